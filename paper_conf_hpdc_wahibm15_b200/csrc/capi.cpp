// capi.cpp — extern "C" boundary (include/stencilfuse.h) and the executor.
//
// Host code of the transformed program (§5.5.4): the new kernels are
// invoked in the order of the new OEG (plan order).  On several ranks each
// group is preceded by the z-slab halo exchange of the inputs its z-reach
// touches; the group's interior chunks do not depend on the exchange and are
// launched first, so compute overlaps communication.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "sf_internal.h"

stencil_program *sf_program_create_impl(const sp_grid *, int32_t, const sp_array_desc *, int32_t,
                                        const sp_kernel *, sp_comm *);
void sf_plan_set_impl(stencil_program *, int32_t, const int32_t *, const sp_stmt_ref *);
void sf_unfused_prepare(stencil_program *);
sp_comm *sf_comm_create_impl(const void *, int32_t, int32_t);
void sf_comm_destroy_impl(sp_comm *);
void sf_comm_unique_id_impl(void *);
void sf_comm_create_loopback_impl(int32_t, sp_comm **);
void sf_ipc_export_impl(const void *, void *, int64_t *);
void *sf_ipc_open_impl(const void *, int64_t);

namespace sf {
static thread_local std::string t_err;
void set_error(const std::string &m) { t_err = m; }
void fail(sp_status code, const std::string &msg) { throw Error{code, msg}; }
}  // namespace sf

using namespace sf;

template <class F>
static sp_status guard(F &&f) {
    try {
        f();
        t_err.clear();
        return SP_OK;
    } catch (const Error &e) {
        t_err = e.msg;
        return e.code;
    } catch (const std::bad_alloc &) {
        t_err = "out of host memory";
        return SP_E_RESOURCES;
    } catch (const std::exception &e) {
        t_err = e.what();
        return SP_E_ARG;
    } catch (...) {
        t_err = "unknown error";
        return SP_E_ARG;
    }
}

static Mode &mode_of(stencil_program *p, int mode) {
    if (mode == 0) {
        sf_unfused_prepare(p);
        return p->unfused;
    }
    if (mode == 1) {
        if (!p->has_plan) fail(SP_E_STATE, "no fusion plan set");
        return p->fused;
    }
    fail(SP_E_ARG, "mode must be 0 (unfused) or 1 (fused)");
}

// output planes [*zb, *ze) of launch L that read no ghost plane received by the
// exchange in front of it: they run while the exchange is in flight
static void interior_planes(const stencil_program *p, const Launch &L,
                            const std::vector<Mode::Xfer> &x, int *zb, int *ze) {
    const int nz = (int)p->grid.nz_local;
    int b = 0, e = nz;
    for (const Mode::Xfer &t : x)
        for (const Input &I : L.in)
            if (I.arr == t.arr) {
                b = std::max(b, -I.qlo);
                e = std::min(e, nz - std::max(0, I.ahi));
            }
    *zb = b;
    *ze = e;
}

// ---------------------------------------------------------------- z-wave schedule
// The step is cut into waves of S planes; in wave w launch i covers planes
// [w*S - off_i, (w+1)*S - off_i).  The skew off_i makes every wave of a launch
// independent of later waves of earlier launches:
//   RAW  (j < i stores X, i reads X up to ahi planes above its chunk):  off_i >= off_j + ahi
//   WAR  (j < i, j reads X down to qlo planes below its chunk, i stores X): off_i >= off_j - qlo
//   WAW  (j < i both store X): off_i >= off_j
// so the result is the plan's result (bit-exact: every point is evaluated by the
// same code, only the chunking changes, P6).  Consecutive launches of one wave
// touch the same few-MB z-slab, so a producer's output is still in the 126 MB L2
// when its consumer reads it (cross-group locality the paper gets from fusion).
static void wave_offsets(const stencil_program *p, Mode &m) {
    const size_t n = m.launches.size();
    m.wave_off.assign(n, 0);
    std::vector<std::vector<int>> stores(n);
    for (size_t i = 0; i < n; ++i)
        for (const Stage &G : m.launches[i].st)
            if (G.stored) stores[i].push_back(G.out);
    auto stores_arr = [&](size_t i, int a) {
        return std::find(stores[i].begin(), stores[i].end(), a) != stores[i].end();
    };
    for (size_t i = 0; i < n; ++i) {
        if (m.launches[i].dead) continue;
        int off = 0;
        for (size_t j = 0; j < i; ++j) {
            if (m.launches[j].dead) continue;
            for (const Input &I : m.launches[i].in)
                if (stores_arr(j, I.arr)) off = std::max(off, m.wave_off[j] + std::max(0, I.ahi));
            for (const Input &I : m.launches[j].in)
                if (stores_arr(i, I.arr)) off = std::max(off, m.wave_off[j] + std::max(0, -I.qlo));
            for (int a : stores[i])
                if (stores_arr(j, a)) off = std::max(off, m.wave_off[j]);
        }
        m.wave_off[i] = off;
    }
    (void)p;
}

static void run_waves(stencil_program *p, Mode &m, void *stream) {
    if (m.wave_off.size() != m.launches.size()) wave_offsets(p, m);
    const int S = p->opt.zwave, ns = std::max(1, p->opt.zwave_streams);
    const int nz = (int)p->grid.nz_local, n = (int)m.launches.size();
    int maxoff = 0;
    for (int o : m.wave_off) maxoff = std::max(maxoff, o);
    const int nw = (nz + maxoff + S - 1) / S;
    auto range = [&](int w, int i, int *z0, int *z1) {
        *z0 = std::max(0, w * S - m.wave_off[i]);
        *z1 = std::min(nz, (w + 1) * S - m.wave_off[i]);
        return *z1 > *z0;
    };
    auto go = [&](int w, int i, void *s) {
        int z0, z1;
        if (m.launches[i].dead || !range(w, i, &z0, &z1)) return false;
        launch(p, m, i, s, z0, z1);
        return true;
    };
    if (ns == 1) {
        for (int w = 0; w < nw; ++w)
            for (int i = 0; i < n; ++i) go(w, i, stream);
        return;
    }
    // ns streams, wave w on stream w % ns; (w, i) waits on (w-1, i) (and, by stream
    // order, on (w, j < i)): the skew keeps everything else that may run
    // concurrently (waves w-1.. of later launches) on disjoint planes
    while ((int)p->wave_streams.size() < ns) {
        cudaStream_t s;
        if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess)
            fail(SP_E_CUDA, "cudaStreamCreate");
        p->wave_streams.push_back(s);
    }
    const size_t nev = (size_t)ns * n + 1 + ns;
    while (p->wave_events.size() < nev) {
        cudaEvent_t ev;
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess)
            fail(SP_E_CUDA, "cudaEventCreate");
        p->wave_events.push_back(ev);
    }
    auto ev = [&](size_t k) { return (cudaEvent_t)p->wave_events[k]; };
    auto st = [&](int k) { return (cudaStream_t)p->wave_streams[k]; };
    const size_t fork = (size_t)ns * n, join0 = fork + 1;
    if (cudaEventRecord(ev(fork), (cudaStream_t)stream) != cudaSuccess)
        fail(SP_E_CUDA, "event record");
    for (int k = 0; k < ns; ++k)
        if (cudaStreamWaitEvent(st(k), ev(fork), 0) != cudaSuccess) fail(SP_E_CUDA, "stream wait");
    std::vector<char> prev(n, 0), cur(n, 0);
    for (int w = 0; w < nw; ++w) {
        cudaStream_t s = st(w % ns);
        for (int i = 0; i < n; ++i) {
            if (prev[i] && cudaStreamWaitEvent(s, ev((size_t)((w - 1) % ns) * n + i), 0) != cudaSuccess)
                fail(SP_E_CUDA, "stream wait");
            cur[i] = go(w, i, s);
            if (cur[i] && cudaEventRecord(ev((size_t)(w % ns) * n + i), s) != cudaSuccess)
                fail(SP_E_CUDA, "event record");
        }
        prev.swap(cur);
    }
    for (int k = 0; k < ns; ++k) {
        if (cudaEventRecord(ev(join0 + k), st(k)) != cudaSuccess ||
            cudaStreamWaitEvent((cudaStream_t)stream, ev(join0 + k), 0) != cudaSuccess)
            fail(SP_E_CUDA, "event record/wait");
    }
}

// kernel launches one run_* call issues under the current communicator and options
// (mirrors run_mode / run_waves: a launch that receives ghost planes on several
// ranks is an interior launch plus one two-range boundary launch, or one launch
// when its interior is empty)
static int count_launches(stencil_program *p, int mode) {
    Mode &m = mode_of(p, mode);
    const bool multi = p->comm && p->comm->nranks > 1;
    const int nz = (int)p->grid.nz_local;
    int n = 0;
    if (mode == 1 && p->opt.zwave > 0 && !multi) {
        if (m.wave_off.size() != m.launches.size()) wave_offsets(p, m);
        const int S = p->opt.zwave;
        int maxoff = 0;
        for (int o : m.wave_off) maxoff = std::max(maxoff, o);
        const int nw = (nz + maxoff + S - 1) / S;
        for (int w = 0; w < nw; ++w)
            for (size_t i = 0; i < m.launches.size(); ++i) {
                if (m.launches[i].dead) continue;
                const int z0 = std::max(0, w * S - m.wave_off[i]);
                const int z1 = std::min(nz, (w + 1) * S - m.wave_off[i]);
                n += z1 > z0;
            }
        return n;
    }
    if (multi && !m.xsched_ok) exchange_schedule(p, m);
    for (size_t i = 0; i < m.launches.size(); ++i) {
        const Launch &L = m.launches[i];
        if (L.dead || L.zc <= 0) continue;
        if (!multi || m.xsched[i].empty()) {
            n += 1;
            continue;
        }
        int zb, ze;
        interior_planes(p, L, m.xsched[i], &zb, &ze);
        n += ze > zb ? 2 : 1;
    }
    return n;
}

// One rank, fused mode, options rename / streams: the launches follow the group DAG on up to
// `streams` streams forked from (and joined back into) the caller's stream; a launch waits
// on the events of its dependencies issued on other streams.  Graph-capturable.
static void run_dag(stencil_program *p, Mode &m, void *stream) {
    dag_analysis(p, m, true);
    prepare_shadows(p, m, stream);  // before the fork: every stream sees initialised shadows
    const int n = (int)m.launches.size();
    int S = 1;
    for (int s : m.stream_of) S = std::max(S, s + 1);
    while ((int)p->dag_streams.size() < S - 1) {
        cudaStream_t s;
        int lo = 0, hi = 0;  // numerically: lo = least priority (0), hi = greatest (negative)
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        const int prio = p->opt.dagprio == 1 ? hi : p->opt.dagprio == 2 ? lo : 0;
        if (cudaStreamCreateWithPriority(&s, cudaStreamNonBlocking, prio) != cudaSuccess)
            fail(SP_E_CUDA, "cudaStreamCreate");
        p->dag_streams.push_back(s);
    }
    while ((int)p->dag_events.size() < n + S) {
        cudaEvent_t ev;
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess)
            fail(SP_E_CUDA, "cudaEventCreate");
        p->dag_events.push_back(ev);
    }
    auto st = [&](int s) { return s == 0 ? (cudaStream_t)stream : (cudaStream_t)p->dag_streams[s - 1]; };
    auto ev = [&](int k) { return (cudaEvent_t)p->dag_events[k]; };
    if (S > 1) {  // fork
        if (cudaEventRecord(ev(n), st(0)) != cudaSuccess) fail(SP_E_CUDA, "event record");
        for (int s = 1; s < S; ++s)
            if (cudaStreamWaitEvent(st(s), ev(n), 0) != cudaSuccess) fail(SP_E_CUDA, "stream wait");
    }
    for (int i = 0; i < n; ++i) {
        const int s = m.stream_of[i];
        for (int d : m.deps[i])
            if (m.stream_of[d] != s && cudaStreamWaitEvent(st(s), ev(d), 0) != cudaSuccess)
                fail(SP_E_CUDA, "stream wait");
        launch(p, m, i, st(s));
        if (S > 1 && cudaEventRecord(ev(i), st(s)) != cudaSuccess) fail(SP_E_CUDA, "event record");
    }
    for (int s = 1; s < S; ++s) {  // join
        if (cudaEventRecord(ev(n + s), st(s)) != cudaSuccess ||
            cudaStreamWaitEvent(st(0), ev(n + s), 0) != cudaSuccess)
            fail(SP_E_CUDA, "event join");
    }
}

static void run_mode(stencil_program *p, int mode, void *stream) {
    Mode &m = mode_of(p, mode);
    load_mode(p, m);
    const bool multi = p->comm && p->comm->nranks > 1;
    if (mode == 1 && p->opt.zwave > 0 && !multi) {
        run_waves(p, m, stream);
        return;
    }
    if (!multi && mode == 1 && (p->opt.rename || p->opt.streams > 1)) {
        run_dag(p, m, stream);
        return;
    }
    if (!multi) {
        for (size_t i = 0; i < m.launches.size(); ++i) launch(p, m, (int)i, stream);
        return;
    }
    // several ranks: programmatic dependent launch is not used across the exchange's
    // events (launch() sees p->no_pdl); each launch whose schedule receives ghost
    // planes runs its interior planes while the exchange is in flight, then the
    // boundary planes (a few planes each) once the ghosts have arrived
    if (!m.xsched_ok) exchange_schedule(p, m);
    p->no_pdl = true;
    const int nz = (int)p->grid.nz_local;
    cudaStream_t cs = (cudaStream_t)comm_stream(p->comm);
    while (p->events.size() < 2) {
        cudaEvent_t ev;
        if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess)
            fail(SP_E_CUDA, "cudaEventCreate");
        p->events.push_back(ev);
    }
    cudaEvent_t ready = (cudaEvent_t)p->events[0], done = (cudaEvent_t)p->events[1];
    auto planes = [&](int i, int z0, int z1, int z2 = 0, int z3 = 0) {
        launch(p, m, i, stream, z0, z1, z2, z3);
    };
    for (size_t i = 0; i < m.launches.size(); ++i) {
        Launch &L = m.launches[i];
        if (L.dead) continue;
        const std::vector<Mode::Xfer> &x = m.xsched[i];
        if (x.empty()) {
            planes((int)i, 0, nz);
            continue;
        }
        int zb, ze;
        interior_planes(p, L, x, &zb, &ze);
        // exchange on the communicator's stream, ordered after prior work on `stream`
        if (cudaEventRecord(ready, (cudaStream_t)stream) != cudaSuccess ||
            cudaStreamWaitEvent(cs, ready, 0) != cudaSuccess)
            fail(SP_E_CUDA, "event record/wait");
        exchange(p, x, cs);
        if (cudaEventRecord(done, cs) != cudaSuccess) fail(SP_E_CUDA, "event record");
        const bool split = ze > zb;
        if (split) planes((int)i, zb, ze);  // interior: overlaps the exchange
        if (cudaStreamWaitEvent((cudaStream_t)stream, done, 0) != cudaSuccess)
            fail(SP_E_CUDA, "stream wait");
        if (split) {
            planes((int)i, 0, zb, ze, nz);  // both boundary ranges in one launch
        } else {
            planes((int)i, 0, nz);
        }
    }
}

extern "C" {

const char *sp_last_error(void) { return t_err.c_str(); }

sp_status sp_comm_unique_id(void *out128) {
    return guard([&] {
        if (!out128) fail(SP_E_ARG, "null output");
        sf_comm_unique_id_impl(out128);
    });
}

sp_status sp_comm_create(const void *id, int32_t nranks, int32_t rank, sp_comm **out) {
    return guard([&] {
        if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks) fail(SP_E_ARG, "bad comm args");
        *out = sf_comm_create_impl(id, nranks, rank);
    });
}

sp_status sp_comm_create_loopback(int32_t nranks, sp_comm **out) {
    return guard([&] {
        if (!out || nranks < 1) fail(SP_E_ARG, "bad loopback args");
        sf_comm_create_loopback_impl(nranks, out);
    });
}

void sp_comm_destroy(sp_comm *c) {
    if (c) guard([&] { sf_comm_destroy_impl(c); });
}

sp_status stencil_program_create(const sp_grid *grid, int32_t n_arrays, const sp_array_desc *arrays,
                                 int32_t n_kernels, const sp_kernel *kernels, sp_comm *comm,
                                 stencil_program **out) {
    return guard([&] {
        if (!out) fail(SP_E_ARG, "null output pointer");
        *out = nullptr;
        *out = sf_program_create_impl(grid, n_arrays, arrays, n_kernels, kernels, comm);
    });
}

void stencil_program_destroy(stencil_program *p) {
    if (!p) return;
    guard([&] {
        unload_mode(p->unfused);
        unload_mode(p->fused);
        for (void *e : p->events) cudaEventDestroy((cudaEvent_t)e);
        for (void *e : p->wave_events) cudaEventDestroy((cudaEvent_t)e);
        for (void *s : p->wave_streams) cudaStreamDestroy((cudaStream_t)s);
        for (void *e : p->dag_events) cudaEventDestroy((cudaEvent_t)e);
        for (void *s : p->dag_streams) cudaStreamDestroy((cudaStream_t)s);
        for (auto &v : p->shadow)
            for (void *q : v) cudaFree(q);
        if (p->sig) cudaFree(p->sig);
    });
    delete p;
}

sp_status stencil_program_layout(const stencil_program *p, sp_layout *out) {
    return guard([&] {
        if (!p || !out) fail(SP_E_ARG, "null argument");
        *out = p->layout;
    });
}

sp_status stencil_program_bind(stencil_program *p, int32_t array, void *dev_ptr) {
    return guard([&] {
        if (!p || array < 0 || array >= (int)p->arrays.size()) fail(SP_E_ARG, "bad array index");
        if (!dev_ptr || ((uintptr_t)dev_ptr & 255))
            fail(SP_E_ARG, "device pointer must be non-null and 256-byte aligned");
        if (p->ptrs[array] != dev_ptr) {
            p->ptrs[array] = dev_ptr;
            p->bind_version++;
        }
    });
}

sp_status sp_signal_buffer(stencil_program *p, void **out) {
    return guard([&] {
        if (!p || !out) fail(SP_E_ARG, "null argument");
        *out = signal_block(p);
    });
}

sp_status sp_bind_peer(stencil_program *p, int32_t array, int32_t side, void *peer_ptr) {
    return guard([&] {
        if (!p || array < 0 || array >= (int)p->arrays.size() || side < 0 || side > 1)
            fail(SP_E_ARG, "bad array index or side");
        if (peer_ptr && ((uintptr_t)peer_ptr & 255)) fail(SP_E_ARG, "peer pointer must be 256-byte aligned");
        p->peer[array][side] = peer_ptr;
        p->bind_version++;
    });
}

sp_status sp_bind_peer_signal(stencil_program *p, int32_t side, void *peer_signal) {
    return guard([&] {
        if (!p || side < 0 || side > 1) fail(SP_E_ARG, "bad side");
        p->peer_sig[side] = peer_signal;
        p->bind_version++;
    });
}

sp_status sp_ipc_export(const void *dev_ptr, void *handle64, int64_t *offset) {
    return guard([&] {
        if (!dev_ptr || !handle64 || !offset) fail(SP_E_ARG, "null argument");
        ensure_cuda();
        sf_ipc_export_impl(dev_ptr, handle64, offset);
    });
}

sp_status sp_ipc_open(const void *handle64, int64_t offset, void **dev_ptr) {
    return guard([&] {
        if (!handle64 || !dev_ptr || offset < 0) fail(SP_E_ARG, "bad argument");
        ensure_cuda();
        *dev_ptr = sf_ipc_open_impl(handle64, offset);
    });
}

sp_status sp_program_set_option(stencil_program *p, const char *key, int64_t v) {
    return guard([&] {
        if (!p || !key) fail(SP_E_ARG, "null argument");
        std::string k = key;
        Options &o = p->opt;
        if (k == "fmad") o.fmad = v != 0;
        else if (k == "tile_x") o.tile_x = (int)v;
        else if (k == "tile_y") o.tile_y = (int)v;
        else if (k == "zchunk") o.zchunk = (int)v;
        else if (k == "threads") o.threads = (int)v;
        else if (k == "prefetch") o.prefetch = (int)v;
        else if (k == "num_sms") p->num_sms = (int)v;
        else if (k == "loader") o.loader = (int)v;
        else if (k == "block_x") o.block_x = (int)v;
        else if (k == "block_y") o.block_y = (int)v;
        else if (k == "block_cby") o.block_cby = (int)v;
        else if (k == "zqueue") o.zqueue = (int)v;
        else if (k == "suspend_hint") o.suspend_hint = (int)v;
        else if (k == "coef_const") o.coef_const = (int)v;
        else if (k == "l2pf") o.l2pf = (int)v;
        else if (k == "pdl") o.pdl = std::max(0, std::min(2, (int)v));
        else if (k == "acc_split") o.acc_split = std::max(1, std::min(4, (int)v));
        else if (k == "factor") o.factor = v != 0;
        else if (k == "zwave") o.zwave = (int)v;
        else if (k == "zwave_streams") o.zwave_streams = std::max(1, std::min(8, (int)v));
        else if (k == "xpush") o.xpush = v != 0;
        else if (k == "fastpath") o.fastpath = (int)std::min<int64_t>(v, 2);
        else if (k == "cluster_x") o.cluster_x = (int)std::max<int64_t>(1, std::min<int64_t>(v, 8));
        else if (k == "minblocks") o.minblocks = (int)std::max<int64_t>(1, std::min<int64_t>(v, 32));
        else if (k == "regcap") o.regcap = (int)std::min<int64_t>(v, 2);
        else if (k == "halo_sel") o.halo_sel = v != 0;
        else if (k == "frame") o.frame = (int)std::min<int64_t>(v, 2);
        else if (k == "psleep") o.psleep = (int)std::min<int64_t>(v, 10000);
        else if (k == "phint") o.phint = (int)std::min<int64_t>(v, 1000000);
        else if (k == "pow2ring") o.pow2ring = v != 0;
        else if (k == "pbar") o.pbar = v != 0;
        else if (k == "rename") o.rename = v != 0;
        else if (k == "streams") o.streams = (int)std::max<int64_t>(1, std::min<int64_t>(v, 8));
        else if (k == "dagprio") o.dagprio = (int)std::min<int64_t>(v, 2);
        else if (k == "dagsched") o.dagsched = (int)std::min<int64_t>(v, 1);
        else if (k == "l2_flush") {}
        else fail(SP_E_ARG, "unknown option '" + k + "'");
        if (v < 0 && k != "prefetch") fail(SP_E_ARG, "negative option value");
        if ((k == "threads" && v && (v % 32 || v > 1024)) || (k == "tile_x" && v > 256) ||
            (k == "tile_y" && v > 256))
            fail(SP_E_ARG, "option value out of range");
        // options change code: drop analysed/compiled state (plans are re-analysed)
        unload_mode(p->unfused);
        p->unfused = Mode();
        if (p->has_plan) {
            Mode m;
            analyze_mode(p, true, p->plan_groups, m);
            unload_mode(p->fused);
            p->fused = std::move(m);
        }
    });
}

sp_status sp_program_counts(const stencil_program *p, int32_t *n_stmts, int32_t *n_edges) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        if (n_stmts) *n_stmts = (int)p->stmts.size();
        if (n_edges) *n_edges = (int)p->edges.size();
    });
}

sp_status sp_program_edges(const stencil_program *p, int32_t cap, sp_edge *out, int32_t *n) {
    return guard([&] {
        if (!p || (cap > 0 && !out)) fail(SP_E_ARG, "null argument");
        int m = std::min<int>(cap, (int)p->edges.size());
        for (int i = 0; i < m; ++i) out[i] = p->edges[i];
        if (n) *n = (int)p->edges.size();
    });
}

sp_status sp_fission_components(const stencil_program *p, int32_t kernel, int32_t *comp,
                                int32_t *n_comp) {
    return guard([&] {
        if (!p || !comp || !n_comp || kernel < 0 || kernel >= (int)p->kernels.size())
            fail(SP_E_ARG, "bad argument");
        int nc = 0;
        std::vector<int> c = fission_components(p, kernel, &nc);
        for (size_t i = 0; i < c.size(); ++i) comp[i] = c[i];
        *n_comp = nc;
    });
}

sp_status fusion_plan_set(stencil_program *p, int32_t n_groups, const int32_t *group_begin,
                          const sp_stmt_ref *members) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        sf_plan_set_impl(p, n_groups, group_begin, members);
    });
}

static void write_plan(const stencil_program *p, const std::vector<std::vector<int>> &gs, int32_t cap,
                       int32_t *n_groups, int32_t *group_begin, sp_stmt_ref *members) {
    *n_groups = (int)gs.size();
    if (!group_begin || !members) return;
    if (cap < (int)gs.size()) fail(SP_E_ARG, "group capacity too small");
    int pos = 0;
    group_begin[0] = 0;
    for (size_t g = 0; g < gs.size(); ++g) {
        for (int gid : gs[g]) {
            const Stmt &S = p->stmts[gid];
            members[pos++] = sp_stmt_ref{S.kernel, S.local};
        }
        group_begin[g + 1] = pos;
    }
}

sp_status sp_plan_greedy(stencil_program *p, int32_t cap, int32_t *n_groups, int32_t *group_begin,
                         sp_stmt_ref *members) {
    return guard([&] {
        if (!p || !n_groups) fail(SP_E_ARG, "null argument");
        write_plan(p, greedy_plan(p), cap, n_groups, group_begin, members);
    });
}

sp_status sp_plan_search(stencil_program *p, int32_t generations, int32_t population, uint64_t seed,
                         int32_t cap, int32_t *n_groups, int32_t *group_begin, sp_stmt_ref *members) {
    return guard([&] {
        if (!p || !n_groups || generations < 0 || population < 1) fail(SP_E_ARG, "bad argument");
        sp_search_options o;
        std::memset(&o, 0, sizeof o);
        o.generations = generations;
        o.population = population;
        o.seed = seed;
        write_plan(p, search_plan(p, o, nullptr, nullptr, nullptr), cap, n_groups, group_begin, members);
    });
}

sp_status sp_plan_search_ex(stencil_program *p, const sp_search_options *opts, sp_stream stream,
                            int32_t cap, int32_t *n_groups, int32_t *group_begin, sp_stmt_ref *members,
                            sp_tile_config *configs, sp_search_report *report) {
    return guard([&] {
        if (!p || !opts || !n_groups || opts->generations < 0 || opts->population < 0 ||
            opts->objective < 0 || opts->objective > 1 || opts->n_configs < 0 ||
            (opts->n_configs > 0 && !opts->configs))
            fail(SP_E_ARG, "bad argument");
        std::vector<sp_tile_config> cfgs;
        const auto gs = search_plan(p, *opts, stream, report, &cfgs);
        write_plan(p, gs, cap, n_groups, group_begin, members);
        if (configs && group_begin)
            for (size_t g = 0; g < gs.size(); ++g) configs[g] = cfgs[g];
    });
}

sp_status sp_plan_count(const stencil_program *p, int32_t mode, int32_t *n) {
    return guard([&] {
        if (!p || !n) fail(SP_E_ARG, "null argument");
        *n = (int)mode_of(const_cast<stencil_program *>(p), mode).launches.size();
    });
}

sp_status sp_plan_report(const stencil_program *p, int32_t mode, int32_t i, sp_group_report *out) {
    return guard([&] {
        if (!p || !out) fail(SP_E_ARG, "null argument");
        Mode &m = mode_of(const_cast<stencil_program *>(p), mode);
        if (i < 0 || i >= (int)m.launches.size()) fail(SP_E_ARG, "launch index out of range");
        fill_report(p, m.launches[i], out);
    });
}

sp_status fusion_plan_report(const stencil_program *p, int32_t group, sp_group_report *out) {
    return sp_plan_report(p, 1, group, out);
}

sp_status sp_plan_source(stencil_program *p, int32_t mode, char *buf, size_t cap, size_t *len) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        Mode &m = mode_of(p, mode);
        std::string all;
        for (const Launch &L : m.launches) all += L.dead ? "// (dead launch " + L.name + ")\n" : L.source;
        if (len) *len = all.size();
        if (buf && cap) {
            size_t n = std::min(cap - 1, all.size());
            std::memcpy(buf, all.data(), n);
            buf[n] = 0;
        }
    });
}

sp_status sp_plan_tune(stencil_program *p, int32_t mode, int32_t launch, const sp_tile_config *cfg) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        Mode &m = mode_of(p, mode);
        if (launch < 0 || launch >= (int)m.launches.size()) fail(SP_E_ARG, "launch index out of range");
        auto &tune = mode ? p->tune_fused : p->tune_unfused;
        auto saved = tune;
        if (cfg) tune[launch] = *cfg;
        else tune.erase(launch);
        Mode n;
        try {
            if (mode) analyze_mode(p, true, p->plan_groups, n);
            else {
                std::vector<std::vector<int>> groups;
                for (const Kernel &K : p->kernels) groups.push_back(K.stmts);
                analyze_mode(p, false, groups, n);
            }
        } catch (...) {
            tune = saved;
            throw;
        }
        unload_mode(m);
        m = std::move(n);
    });
}

sp_status sp_plan_exchange(stencil_program *p, int32_t mode, int32_t launch, int32_t cap,
                           int32_t *arrays, int32_t *below, int32_t *above, int32_t *n) {
    return guard([&] {
        if (!p || !n || (cap > 0 && !arrays)) fail(SP_E_ARG, "null argument");
        Mode &m = mode_of(p, mode);
        if (launch < 0 || launch >= (int)m.launches.size()) fail(SP_E_ARG, "launch index out of range");
        if (!m.xsched_ok) exchange_schedule(p, m);
        const std::vector<Mode::Xfer> &x = m.xsched[launch];
        *n = (int)x.size();
        for (int i = 0; i < std::min<int>(cap, (int)x.size()); ++i) {
            arrays[i] = x[i].arr;
            if (below) below[i] = x[i].below;
            if (above) above[i] = x[i].above;
        }
    });
}

sp_status sp_plan_wave_offsets(stencil_program *p, int32_t cap, int32_t *off, int32_t *n) {
    return guard([&] {
        if (!p || !n || (cap > 0 && !off)) fail(SP_E_ARG, "null argument");
        Mode &m = mode_of(p, 1);
        wave_offsets(p, m);
        *n = (int)m.wave_off.size();
        for (int i = 0; i < std::min<int>(cap, *n); ++i) off[i] = m.wave_off[i];
    });
}

sp_status sp_compile(stencil_program *p, int32_t mode) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        compile_mode(p, mode_of(p, mode));
    });
}

sp_status sp_load(stencil_program *p, int32_t mode) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        load_mode(p, mode_of(p, mode));
    });
}

sp_status run_unfused(stencil_program *p, sp_stream stream) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        run_mode(p, 0, stream);
    });
}

sp_status run_fused(stencil_program *p, sp_stream stream) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        run_mode(p, 1, stream);
    });
}

sp_status sp_run_launch(stencil_program *p, int32_t mode, int32_t i, sp_stream stream) {
    return guard([&] {
        if (!p) fail(SP_E_ARG, "null program");
        Mode &m = mode_of(p, mode);
        if (i < 0 || i >= (int)m.launches.size()) fail(SP_E_ARG, "launch index out of range");
        load_mode(p, m);
        if (p->comm && p->comm->nranks > 1) p->no_pdl = true;
        launch(p, m, i, stream);
    });
}

sp_status sp_run_launch_count(stencil_program *p, int32_t mode, int32_t *n) {
    return guard([&] {
        if (!p || !n) fail(SP_E_ARG, "null argument");
        *n = count_launches(p, mode);
    });
}

sp_status sp_plan_dag(stencil_program *p, int32_t mode, int32_t launch, int32_t cap, int32_t *deps,
                      int32_t *n_deps, int32_t *stream) {
    return guard([&] {
        if (!p || !n_deps || !stream || (cap > 0 && !deps)) fail(SP_E_ARG, "null argument");
        Mode &m = mode_of(p, mode);
        if (launch < 0 || launch >= (int)m.launches.size()) fail(SP_E_ARG, "bad launch index");
        dag_analysis(p, m, mode == 1);
        const std::vector<int> &d = m.deps[launch];
        for (int k = 0; k < std::min<int>(cap, (int)d.size()); ++k) deps[k] = d[k];
        *n_deps = (int)d.size();
        *stream = m.stream_of[launch];
    });
}

sp_status exchange_halos(stencil_program *p, int32_t n, const int32_t *arrays, int32_t depth,
                         sp_stream stream) {
    return guard([&] {
        if (!p || n < 0 || (n > 0 && !arrays)) fail(SP_E_ARG, "bad argument");
        if (!p->comm) fail(SP_E_STATE, "exchange_halos needs a communicator");
        if (depth < 1 || depth > p->grid.zhalo || depth > p->grid.nz_local)
            fail(SP_E_ARG, "depth must be in [1, min(zhalo, nz_local)]");
        std::vector<Mode::Xfer> x;
        for (int i = 0; i < n; ++i) {
            if (arrays[i] < 0 || arrays[i] >= (int)p->arrays.size()) fail(SP_E_ARG, "bad array index");
            x.push_back({arrays[i], depth, depth});
        }
        exchange(p, x, stream);
    });
}

}  // extern "C"
