// jit.cpp — NVRTC compilation for sm_100a, module loading, TMA descriptors, launches.
//
// The generated kernels ("code generation", §3.2.5 and P:L278-296
// §5.5) are compiled at run time: the program description is the input, so
// there is no CUDA source to rewrite (the paper's ROSE path).  Each
// launch is its own NVRTC program, compiled in parallel host threads; cubins
// are cached in-process by source hash.  Driver entry points come through the
// runtime (cudaGetDriverEntryPoint), so the library loads on hosts without a
// GPU and fails with SP_E_CUDA only when a device call is made.
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvrtc.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <thread>
#include <unordered_map>

#include "sf_internal.h"

namespace sf {

static const char *kDeviceHeader =
#include "sf_device_embed.inc"
    ;

struct Drv {
    CUresult (*ModuleLoadData)(CUmodule *, const void *) = nullptr;
    CUresult (*ModuleUnload)(CUmodule) = nullptr;
    CUresult (*ModuleGetFunction)(CUfunction *, CUmodule, const char *) = nullptr;
    CUresult (*FuncSetAttribute)(CUfunction, CUfunction_attribute, int) = nullptr;
    CUresult (*FuncGetAttribute)(int *, CUfunction_attribute, CUfunction) = nullptr;
    CUresult (*LaunchKernel)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned,
                             unsigned, unsigned, CUstream, void **, void **) = nullptr;
    CUresult (*TensorMapEncodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                     const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                     const cuuint32_t *, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion,
                                     CUtensorMapFloatOOBfill) = nullptr;
    CUresult (*GetErrorString)(CUresult, const char **) = nullptr;
    CUresult (*LaunchKernelEx)(const CUlaunchConfig *, CUfunction, void **, void **) = nullptr;
    CUresult (*MemGetAddressRange)(CUdeviceptr *, size_t *, CUdeviceptr) = nullptr;
    std::atomic<bool> ok{false};
};
static Drv g_drv;
static std::mutex g_drv_mu;

static void cuda_check(cudaError_t e, const char *what) {
    if (e != cudaSuccess)
        fail(SP_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

static void drv_check(CUresult r, const char *what) {
    if (r != CUDA_SUCCESS) {
        const char *s = "unknown";
        if (g_drv.GetErrorString) g_drv.GetErrorString(r, &s);
        fail(SP_E_CUDA, std::string(what) + ": " + s);
    }
}

template <class F>
static void entry(const char *name, F &fp) {
    void *ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint(name, &ptr, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !ptr)
        fail(SP_E_CUDA, std::string("driver entry point ") + name + " unavailable");
    fp = reinterpret_cast<F>(ptr);
}

void ensure_cuda() {
    // fast path: no runtime call (cudaFree(0) may synchronize the device, which a
    // rank whose kernels wait on a neighbour's progress must never do mid-step)
    if (g_drv.ok) return;
    std::lock_guard<std::mutex> lk(g_drv_mu);
    if (g_drv.ok) return;
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0)
        fail(SP_E_CUDA, std::string("no CUDA device available (") + cudaGetErrorString(e) +
                            "); this library has no CPU fallback");
    cuda_check(cudaFree(nullptr), "cudaFree(0) (context init)");
    entry("cuModuleLoadData", g_drv.ModuleLoadData);
    entry("cuModuleUnload", g_drv.ModuleUnload);
    entry("cuModuleGetFunction", g_drv.ModuleGetFunction);
    entry("cuFuncSetAttribute", g_drv.FuncSetAttribute);
    entry("cuFuncGetAttribute", g_drv.FuncGetAttribute);
    entry("cuLaunchKernel", g_drv.LaunchKernel);
    entry("cuTensorMapEncodeTiled", g_drv.TensorMapEncodeTiled);
    entry("cuGetErrorString", g_drv.GetErrorString);
    entry("cuLaunchKernelEx", g_drv.LaunchKernelEx);
    entry("cuMemGetAddressRange", g_drv.MemGetAddressRange);
    g_drv.ok = true;
}

bool driver_mem_range(CUdeviceptr *base, size_t *size, CUdeviceptr p) {
    ensure_cuda();
    return g_drv.MemGetAddressRange(base, size, p) == CUDA_SUCCESS;
}

// ------------------------------------------------------------------ NVRTC
static std::mutex g_cache_mu;
static std::unordered_map<std::string, std::pair<std::string, int>> g_cache;  // key -> (cubin, regs)
static std::unordered_map<std::string, int> g_spill;  // key -> spill store bytes

static std::string compile_one(const std::string &src, bool fmad, const std::string &name,
                               int *regs, int maxrreg = 0, int *spill_out = nullptr) {
    std::string key = std::to_string(std::hash<std::string>{}(src)) + (fmad ? "f" : "n") +
                      std::to_string(src.size()) + "r" + std::to_string(maxrreg);
    {
        std::lock_guard<std::mutex> lk(g_cache_mu);
        auto it = g_cache.find(key);
        if (it != g_cache.end()) {
            *regs = it->second.second;
            if (spill_out) *spill_out = g_spill[key];
            return it->second.first;
        }
    }
    nvrtcProgram prog;
    const char *hdr_src[] = {kDeviceHeader};
    const char *hdr_name[] = {"sf_device.cuh"};
    if (nvrtcCreateProgram(&prog, src.c_str(), (name + ".cu").c_str(), 1, hdr_src, hdr_name) !=
        NVRTC_SUCCESS)
        fail(SP_E_JIT, "nvrtcCreateProgram failed");
    std::vector<const char *> opts = {"-arch=sm_100a", "-std=c++17", "-lineinfo",
                                      fmad ? "--fmad=true" : "--fmad=false", "--ftz=false",
                                      "--prec-div=true", "--prec-sqrt=true",
                                      "--ptxas-options=-v", "-DNDEBUG"};
    const std::string mr = "--maxrregcount=" + std::to_string(maxrreg);
    if (maxrreg > 0) opts.push_back(mr.c_str());
    nvrtcResult r = nvrtcCompileProgram(prog, (int)opts.size(), opts.data());
    size_t log_size = 0;
    nvrtcGetProgramLogSize(prog, &log_size);
    std::string log(log_size, '\0');
    if (log_size) nvrtcGetProgramLog(prog, &log[0]);
    if (r != NVRTC_SUCCESS) {
        nvrtcDestroyProgram(&prog);
        fail(SP_E_JIT, "NVRTC failed for " + name + ": " + log.substr(0, 4000));
    }
    size_t n = 0;
    nvrtcGetCUBINSize(prog, &n);
    std::string cubin(n, '\0');
    nvrtcGetCUBIN(prog, &cubin[0]);
    nvrtcDestroyProgram(&prog);
    int rr = -1;
    auto pos = log.find("Used ");
    if (pos != std::string::npos) rr = std::atoi(log.c_str() + pos + 5);
    int spill = 0;
    if (log.find("bytes spill stores") != std::string::npos) {
        auto sp = log.find("bytes spill stores");
        auto b = log.rfind(',', sp);
        spill = std::atoi(log.c_str() + (b == std::string::npos ? 0 : b + 1));
        if (spill > 0 && maxrreg == 0)
            std::fprintf(stderr, "[stencilfuse] warning: %s spills %d bytes\n", name.c_str(), spill);
    }
    *regs = rr;
    if (spill_out) *spill_out = spill;
    if (const char *dir = std::getenv("SF_DUMP_DIR")) {  // debugging aid: source, cubin, log
        std::string base = std::string(dir) + "/" + name;
        if (FILE *f = std::fopen((base + ".cu").c_str(), "w")) { std::fwrite(src.data(), 1, src.size(), f); std::fclose(f); }
        if (FILE *f = std::fopen((base + ".cubin").c_str(), "wb")) { std::fwrite(cubin.data(), 1, cubin.size(), f); std::fclose(f); }
        if (FILE *f = std::fopen((base + ".log").c_str(), "w")) { std::fwrite(log.data(), 1, log.size(), f); std::fclose(f); }
    }
    std::lock_guard<std::mutex> lk(g_cache_mu);
    g_cache[key] = {cubin, rr};
    g_spill[key] = spill;
    return cubin;
}

// Resident CTAs per SM of a launch as the hardware allocates them: registers per
// warp in units of 256, each of the 4 SM sub-partitions holding 16K registers and
// a quarter of the resident warps (ceil); shared memory 228 KB with 1 KB reserved
// per CTA; at most 64 warps and 32 CTAs.  Measured on B200 (ncu occupancy limits):
// 160-thread CTAs fit 3 per SM at 128 registers and 2 at 132.
static int resident_ctas(int regs, int nth, int64_t smem, int *by_regs, int *by_rest) {
    const int w = (nth + 31) / 32;
    int rest = std::min<int64_t>({32, 64 / w, (228 * 1024) / (smem + 1024)});
    int rr = 0;
    const int rw = (std::max(regs, 1) * 32 + 255) / 256 * 256;
    for (int c = 1; c <= 32; ++c)
        if (((c * w + 3) / 4) * rw <= 16384) rr = c;
    if (by_regs) *by_regs = rr;
    if (by_rest) *by_rest = rest;
    return std::min(rr, rest);
}

// largest register count that keeps `target` CTAs of nth threads resident
static int regs_for_ctas(int target, int nth) {
    const int w = (nth + 31) / 32;
    const int per_part = (target * w + 3) / 4;
    return std::min(255, 16384 / per_part / 256 * 256 / 32);
}

void compile_mode(stencil_program *p, Mode &m) {
    if (m.compiled) return;
    const int n = (int)m.launches.size();
    std::vector<std::string> errs(n);
    std::atomic<int> next{0};
    auto work = [&]() {
        for (;;) {
            int i = next.fetch_add(1);
            if (i >= n) return;
            Launch &L = m.launches[i];
            if (L.dead) continue;
            try {
                L.cubin = compile_one(L.source, p->opt.fmad != 0, L.fn, &L.regs);
                // occupancy-aware register cap: when the kernel sits a few registers
                // above the budget of one more resident CTA that shared memory would
                // allow, recompile at that budget and keep it if ptxas needs no spills.
                // Default (1): peer-push kernels only, whose protocol adds a few
                // registers to a tuned kernel (C5: 128 -> 132 regs cost a resident CTA
                // and 23 %; capped: 114 regs, back to 3 CTAs/SM); 2: every kernel
                // (measured on the single-GPU C4 step: 1 % slower, so not default)
                int by_regs = 0, by_rest = 0;
                resident_ctas(L.regs, L.nth, L.smem, &by_regs, &by_rest);
                const bool capit = p->opt.regcap == 2 || (p->opt.regcap == 1 && L.xp);
                if (capit && by_regs < by_rest) {
                    const int cap = regs_for_ctas(by_regs + 1, L.nth);
                    if (cap >= 32 && L.regs - cap <= 16) {
                        int r2 = 0, spill = 0;
                        // __launch_bounds__ overrides --maxrregcount and ptxas does not
                        // model the per-sub-partition limit: state the budget directly
                        std::string src2 = L.source;
                        const std::string lb = "__launch_bounds__(" + std::to_string(L.nth) + ", " +
                                               std::to_string(std::max(1, p->opt.minblocks)) + ")";
                        const size_t at = src2.find(lb);
                        if (at != std::string::npos)
                            src2.replace(at, lb.size(), "__maxnreg__(" + std::to_string(cap) + ")");
                        std::string c2 = compile_one(src2, p->opt.fmad != 0, L.fn, &r2, 0, &spill);
                        if (spill == 0 && r2 > 0 && r2 <= cap) {
                            L.cubin = c2;
                            L.regs = r2;
                        }
                    }
                }
            } catch (const Error &e) {
                errs[i] = e.msg;
            }
        }
    };
    int nth = (int)std::min<unsigned>(std::max(1u, std::thread::hardware_concurrency()), 16u);
    nth = std::min(nth, std::max(n, 1));
    std::vector<std::thread> th;
    for (int t = 0; t < nth; ++t) th.emplace_back(work);
    for (auto &t : th) t.join();
    for (int i = 0; i < n; ++i)
        if (!errs[i].empty()) fail(SP_E_JIT, errs[i]);
    m.compiled = true;
}

void unload_mode(Mode &m) {
    if (m.loaded && g_drv.ok)
        for (Launch &L : m.launches)
            if (L.module) g_drv.ModuleUnload((CUmodule)L.module);
    for (Launch &L : m.launches) { L.module = nullptr; L.func = nullptr; }
    m.loaded = false;
}

void load_mode(stencil_program *p, Mode &m) {
    ensure_cuda();
    if (!m.compiled) compile_mode(p, m);
    if (m.loaded) return;
    int dev = 0;
    cuda_check(cudaGetDevice(&dev), "cudaGetDevice");
    int sms = 0;
    cuda_check(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev), "attr");
    for (size_t i = 0; i < m.launches.size(); ++i) {
        Launch &L = m.launches[i];
        if (L.dead) continue;
        CUmodule mod;
        drv_check(g_drv.ModuleLoadData(&mod, L.cubin.data()), "cuModuleLoadData");
        CUfunction f;
        drv_check(g_drv.ModuleGetFunction(&f, mod, L.fn.c_str()), "cuModuleGetFunction");
        drv_check(g_drv.FuncSetAttribute(f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES,
                                         (int)L.smem),
                  "cuFuncSetAttribute(smem)");
        int regs = 0;
        g_drv.FuncGetAttribute(&regs, CU_FUNC_ATTRIBUTE_NUM_REGS, f);
        L.regs = regs;
        L.module = mod;
        L.func = f;
    }
    m.params.assign(m.launches.size(), {});
    m.maps_version = ~0ull;
    m.loaded = true;
}

void *signal_block(stencil_program *p) {
    if (!p->sig) {
        ensure_cuda();
        void *s = nullptr;
        if (cudaMalloc(&s, 64) != cudaSuccess || cudaMemset(s, 0, 64) != cudaSuccess ||
            cudaDeviceSynchronize() != cudaSuccess)
            fail(SP_E_CUDA, "signal block allocation");
        p->sig = s;
    }
    return p->sig;
}

// TEMP instances (option rename): reads of array a in launch i use instance rd_inst[i][a],
// its stores (and the stage's ghost loads: ghost cells are identical in every instance)
// wr_inst[i][a]; instance 0 is the bound buffer
void dag_analysis(stencil_program *p, Mode &m, bool fused) {
    if (m.dag_ok) return;
    const int n = (int)m.launches.size(), na = (int)p->arrays.size();
    const bool multi = p->comm && p->comm->nranks > 1;
    // a z-slab of a decomposed grid (nz_global > nz_local) exchanges ghost planes of the
    // BOUND buffers (the library's schedule or the caller's copies): no renaming there
    const bool slab = p->grid.nz_global != p->grid.nz_local;
    const bool ren = fused && p->opt.rename && !multi && !slab && p->opt.zwave == 0 && p->opt.loader == 0;
    std::vector<bool> renamable(na, false);
    if (ren) {
        for (int a = 0; a < na; ++a) renamable[a] = p->arrays[a].role == SP_TEMP;
        for (const Stmt &S : p->stmts)  // a boxed write keeps the previous values: same buffer
            if (S.boxed) renamable[S.out] = false;
    }
    m.rd_inst.assign(n, std::vector<int>(na, 0));
    m.wr_inst.assign(n, std::vector<int>(na, 0));
    m.n_inst.assign(na, 0);
    std::vector<int> cur(na, 0);
    std::vector<bool> written(na, false);
    std::vector<std::set<int>> rd(n), wr(n);  // HBM reads / stores per launch
    for (int i = 0; i < n; ++i) {
        const Launch &L = m.launches[i];
        m.rd_inst[i] = cur;
        if (!L.dead) {
            for (const Input &I : L.in) rd[i].insert(I.arr);
            for (const Stage &G : L.st) {
                if (!G.needed) continue;
                if (p->stmts[G.gid].boxed) rd[i].insert(G.out);  // previous values outside the box
                if (G.stored) wr[i].insert(G.out);
            }
        }
        for (int a : wr[i]) {
            if (renamable[a] && written[a]) cur[a] = ++m.n_inst[a];
            written[a] = true;
        }
        m.wr_inst[i] = cur;
    }
    // dependencies on (array, instance): RAW, WAR, WAW
    m.deps.assign(n, {});
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < i; ++j) {
            bool dep = false;
            for (int a : wr[j]) {
                if (rd[i].count(a) && m.wr_inst[j][a] == m.rd_inst[i][a]) dep = true;
                if (wr[i].count(a) && m.wr_inst[j][a] == m.wr_inst[i][a]) dep = true;
            }
            for (int a : rd[j])
                if (wr[i].count(a) && m.rd_inst[j][a] == m.wr_inst[i][a]) dep = true;
            if (dep) m.deps[i].push_back(j);
        }
    // streams: a launch follows its latest dependency's stream, else the least-loaded one
    const int S = (fused && !multi && p->opt.zwave == 0) ? std::max(1, p->opt.streams) : 1;
    m.stream_of.assign(n, 0);
    std::vector<int> load(S, 0);
    for (int i = 0; i < n; ++i) {
        int s = 0;
        if (p->opt.dagsched == 1 && S > 1)  // roots (no dependency) run ahead on the last stream
            s = m.deps[i].empty() ? S - 1 : 0;
        else if (!m.deps[i].empty()) s = m.stream_of[m.deps[i].back()];
        else s = (int)(std::min_element(load.begin(), load.end()) - load.begin());
        m.stream_of[i] = s;
        load[s] += m.launches[i].dead ? 0 : 1;
    }
    m.dag_ok = true;
}

static void *inst_ptr(stencil_program *p, int a, int inst) {
    if (inst == 0) return p->ptrs[a];
    return p->shadow[a][inst - 1];
}

void prepare_shadows(stencil_program *p, Mode &m, void *stream) {
    const int na = (int)p->arrays.size();
    if ((int)p->shadow.size() < na) p->shadow.resize(na);
    if ((int)m.shadow_src.size() < na) m.shadow_src.assign(na, nullptr);
    for (int a = 0; a < na; ++a) {
        const int k = m.n_inst.empty() ? 0 : m.n_inst[a];
        if (!k) continue;
        if (!p->ptrs[a]) fail(SP_E_STATE, "array '" + p->arrays[a].name + "' is not bound");
        // only a TEMP whose bound buffer changed needs its shadows (re)initialised: rebinding
        // other arrays every step (double-buffered inputs) costs nothing here
        if (m.shadow_src[a] == p->ptrs[a] && (int)p->shadow[a].size() >= k) continue;
        while ((int)p->shadow[a].size() < k) {
            void *q = nullptr;
            if (cudaMalloc(&q, (size_t)p->layout.bytes) != cudaSuccess)
                fail(SP_E_CUDA, "shadow buffer of '" + p->arrays[a].name + "' (option rename)");
            p->shadow[a].push_back(q);
        }
        // the ghost cells every instance must carry (reading R1): a copy of the bound buffer
        for (int j = 0; j < k; ++j)
            cuda_check(cudaMemcpyAsync(p->shadow[a][j], p->ptrs[a], (size_t)p->layout.bytes,
                                       cudaMemcpyDeviceToDevice, (cudaStream_t)stream),
                       "shadow init copy");
        m.shadow_src[a] = p->ptrs[a];
    }
}

static void build_params(stencil_program *p, Mode &m) {
    if (m.maps_version == p->bind_version) return;
    const bool inst = m.dag_ok && !m.rd_inst.empty();
    const int e = p->elem;
    const sp_layout &lay = p->layout;
    for (size_t i = 0; i < m.launches.size(); ++i) {
        Launch &L = m.launches[i];
        if (L.dead) continue;
        std::vector<Mode::Blk> &blk = m.params[i];
        blk.assign(L.param_size / 64 + 1, Mode::Blk{});
        unsigned char *buf = blk[0].b;
        for (size_t a = 0; a < L.in.size(); ++a) {
            void *ptr = inst ? inst_ptr(p, L.in[a].arr, m.rd_inst[i][L.in[a].arr]) : p->ptrs[L.in[a].arr];
            if (!ptr) fail(SP_E_STATE, "array '" + p->arrays[L.in[a].arr].name + "' is not bound");
            CUtensorMap tm;
            cuuint64_t dims[3] = {(cuuint64_t)lay.x_pitch, (cuuint64_t)lay.y_alloc,
                                  (cuuint64_t)lay.z_alloc};
            cuuint64_t strides[2] = {(cuuint64_t)(lay.x_pitch * e),
                                     (cuuint64_t)(lay.x_pitch * lay.y_alloc * e)};
            cuuint32_t box[3] = {(cuuint32_t)L.in_rw[a], (cuuint32_t)L.in_rh[a], 1};
            cuuint32_t es[3] = {1, 1, 1};
            drv_check(g_drv.TensorMapEncodeTiled(
                          &tm, e == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                          3, ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE),
                      "cuTensorMapEncodeTiled");
            std::memcpy(buf + 128 * a, &tm, 128);
        }
        for (size_t s = 0; s < L.slot_arr.size(); ++s) {
            void *ptr = inst ? inst_ptr(p, L.slot_arr[s], m.wr_inst[i][L.slot_arr[s]]) : p->ptrs[L.slot_arr[s]];
            if (!ptr) fail(SP_E_STATE, "array '" + p->arrays[L.slot_arr[s]].name + "' is not bound");
            std::memcpy(buf + L.ptr_off + 8 * s, &ptr, 8);
        }
        if (L.xp) {
            // peer-push section: own signal block, neighbours' blocks and buffers
            // (a missing neighbour — rank 0 below, the last rank above — stays null)
            const int r = p->comm->rank, nr = p->comm->nranks;
            const bool has[2] = {r > 0, r + 1 < nr};
            // (allocated by sp_signal_buffer when the peers are wired: allocating here,
            // mid-step, could synchronise the device under a waiting neighbour)
            if (!p->sig) fail(SP_E_STATE, "peer push: no signal block (sp_signal_buffer)");
            char *sig = (char *)p->sig;
            void *v[5] = {sig + 16, sig, has[0] ? p->peer_sig[0] : nullptr,
                          has[1] ? p->peer_sig[1] : nullptr, sig + 24};
            for (int s = 0; s < 2; ++s)
                if (has[s] && !p->peer_sig[s])
                    fail(SP_E_STATE, "peer push: the neighbours' signal blocks are not bound "
                                     "(sp_bind_peer_signal)");
            std::memcpy(buf + L.xp_off, v, 40);
            for (size_t k = 0; k < L.pushes.size(); ++k) {
                const int a = L.st[L.pushes[k].stage].out;
                for (int s = 0; s < 2; ++s) {
                    void *q = has[s] ? p->peer[a][s] : nullptr;
                    if (has[s] && !q)
                        fail(SP_E_STATE, "peer push: neighbour buffer of '" + p->arrays[a].name +
                                             "' is not bound (sp_bind_peer)");
                    std::memcpy(buf + L.xp_off + 40 + 16 * k + 8 * s, &q, 8);
                }
            }
        }
    }
    m.maps_version = p->bind_version;
}

void launch(stencil_program *p, Mode &m, int i, void *stream, int z0, int z1, int z2, int z3) {
    Launch &L = m.launches[i];
    if (L.dead || L.zc <= 0) return;
    const int nz = (int)p->grid.nz_local;
    if (z1 < 0) z1 = nz;
    z0 = std::max(0, z0);
    z1 = std::min(nz, z1);
    z2 = std::max(z2, z1);
    z3 = std::min(z3, nz);
    const int n_lo = z1 > z0 ? (z1 - z0 + L.zc - 1) / L.zc : 0;
    const int n_hi = z3 > z2 ? (z3 - z2 + L.zc - 1) / L.zc : 0;
    const int nchunks = n_lo + n_hi;
    if (nchunks <= 0) return;
    if (&m == &p->fused && (p->opt.rename || p->opt.streams > 1)) dag_analysis(p, m, true);
    if (m.dag_ok && !m.n_inst.empty()) prepare_shadows(p, m, stream);
    build_params(p, m);
    // NVTX range per group launch (SURVEY.md §5 tracing): a tool (Nsight Systems) projects
    // it onto the kernel; a no-op without one attached
    nvtxRangePushA(L.nvtx.c_str());
    struct Pop { ~Pop() { nvtxRangePop(); } } pop_range;
    unsigned char *base = m.params[i][0].b;
    int32_t ints[6] = {n_lo, z1, z2, z0, z3, 0};
    std::memcpy(base + L.int_off, ints, 24);
    void *args[] = {base};
    const bool use_pdl = L.pdl && !p->no_pdl;
    if (use_pdl || L.cx > 1) {
        // programmatic dependent launch: the kernel's prologue may overlap the previous
        // launch on the stream; griddepcontrol.wait in the kernel orders its data accesses.
        // Clusters (option cluster_x): L.cx CTAs along x per cluster
        CUlaunchAttribute attr[2];
        std::memset(attr, 0, sizeof attr);
        int na = 0;
        if (use_pdl) {
            attr[na].id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
            attr[na++].value.programmaticStreamSerializationAllowed = 1;
        }
        if (L.cx > 1) {
            attr[na].id = CU_LAUNCH_ATTRIBUTE_CLUSTER_DIMENSION;
            attr[na].value.clusterDim.x = (unsigned)L.cx;
            attr[na].value.clusterDim.y = 1;
            attr[na++].value.clusterDim.z = 1;
        }
        CUlaunchConfig cfg;
        std::memset(&cfg, 0, sizeof cfg);
        cfg.gridDimX = (unsigned)L.ntx;
        cfg.gridDimY = (unsigned)L.nty;
        cfg.gridDimZ = (unsigned)nchunks;
        cfg.blockDimX = (unsigned)L.nth;
        cfg.blockDimY = cfg.blockDimZ = 1;
        cfg.sharedMemBytes = (unsigned)L.smem;
        cfg.hStream = (CUstream)stream;
        cfg.attrs = attr;
        cfg.numAttrs = (unsigned)na;
        drv_check(g_drv.LaunchKernelEx(&cfg, (CUfunction)L.func, args, nullptr), "cuLaunchKernelEx");
        return;
    }
    drv_check(g_drv.LaunchKernel((CUfunction)L.func, (unsigned)L.ntx, (unsigned)L.nty,
                                 (unsigned)nchunks, (unsigned)L.nth, 1, 1, (unsigned)L.smem,
                                 (CUstream)stream, args, nullptr),
              "cuLaunchKernel");
}

}  // namespace sf
