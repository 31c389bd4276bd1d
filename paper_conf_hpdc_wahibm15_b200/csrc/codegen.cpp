// codegen.cpp — emits the CUDA source of one launch (fused group or original kernel).
//
// The kernel is a 2.5-D z-march (horizontal mapping to the CUDA
// grid, iteration in the vertical direction): one CTA owns a TX x TY tile and a
// chunk of ZC planes.  Warp roles:
//   * producer warp (last warp, one lane): per step j it issues one batch of TMA
//     loads — for every input the plane first needed at step j — into that
//     input's shared-memory ring, PF steps ahead, gated by a per-step "empty"
//     mbarrier (simple fusion's staging of the arrays "target of locality",
//     P:L288 §5.5.2: every input is read from HBM once per CTA);
//   * compute warps: per step k they wait on the batch's "full" mbarrier,
//     evaluate every statement of the group in program order on its own extended
//     region at its own lead plane k+lead (complex fusion: producer statements on
//     extra halo layers, then a barrier, then consumers on the tile — P:L292
//     §5.5.3), store live-out statements on the tile (reading R6) and arrive on
//     the step's empty mbarrier.
//
// Register blocking of the tile core.  Thread (xt, yt) owns CBY blocks of VX x VY
// points: block b covers x in [xt*VX, xt*VX+VX), y in [(b*YT+yt)*VY, +VY).  For a
// statement, every shared-memory value its block needs (all taps of all VX*VY
// points) is loaded once, 16-byte vectorised where aligned; a value needed at
// several planes (z taps) is kept in a register queue that advances one plane
// per step and is refilled by one load of the newest plane.  This divides the
// shared-memory traffic per point — the binding resource of fused stencil
// groups on B200 (SMEM : HBM bandwidth is only ~5.5 : 1) — by the reuse factor.
// Halo strips (the extra layers of complex fusion) are evaluated point-wise.
//
// Region-vector form (option / pin "frame"): instead of register blocks on the tile
// plus point-wise halo strips, every statement is evaluated on its whole extended
// region in units of one 16-byte x-vector, enumerated linearly over the threads
// (unit q = tid + b*NT); the region's x-range is rounded out to the vector
// alignment and the extra lanes compute values no valid point consumes (their reads
// past a row end land in the 128-B guard after every ring plane).  "frame=2" gives all
// statements of a launch one unit grid (the union of their regions), so a unit's
// own-position taps come from per-thread register queues.
//
// Ghost points (reading R1): a point outside the global interior takes the
// array's ghost value through a predicated load; tiles inside the interior skip
// the test.
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <climits>
#include <functional>
#include <set>
#include <sstream>
#include <tuple>

#include "sf_internal.h"

namespace sf {

static std::string lit(double c, bool f32) {
    char buf[64];
    if (f32) std::snprintf(buf, sizeof buf, "%af", (double)(float)c);
    else std::snprintf(buf, sizeof buf, "%a", c);
    return buf;
}

static std::string num(int64_t v) { return std::to_string(v); }
static std::string sg(int v) { return v < 0 ? "m" + num(-v) : "p" + num(v); }

static int log2i(int v) {
    int l = 0;
    while ((1 << l) < v) ++l;
    return l;
}

void core_geometry(const Launch &L, int *xt, int *yt) {
    *xt = L.tx / L.vx;
    *yt = L.nt / *xt;
}

// ------------------------------------------------------------ position analysis
// Values a statement's core block needs: (layout, y, x) relative to the block
// origin, with the range of plane offsets c = lead + dz it is needed at.
struct PosKey {
    bool stage;
    int id, y, x;
    int c = 0;  // plane offset when z-queues are disabled (0 otherwise)
    bool operator<(const PosKey &o) const {
        return std::tie(stage, id, y, x, c) < std::tie(o.stage, o.id, o.y, o.x, o.c);
    }
};
struct PosInfo { int cmin = 1 << 20, cmax = -(1 << 20); };

// z-queue policy: zq 1 = every position read at several planes, per statement;
// zq 2 = input positions inside the block core only (the column a thread owns),
// shared by all statements of the step and refilled once per step
static bool zqueued(const Launch &L, bool stage, int y, int x) {
    if (L.zq == 1) return true;
    return L.zq == 2 && !stage && y >= 0 && y < L.vy && x >= 0 && x < L.vx;
}

static std::map<PosKey, PosInfo> block_positions(const Launch &L, const Stage &G) {
    std::map<PosKey, PosInfo> pos;
    for (const TermR &t : G.terms)
        for (int w = 0; w < 2; ++w) {
            if (w == 1 && !t.has_b) continue;
            const Src &s = w ? t.b : t.a;
            if (s.stage && (L.st[s.idx].keep == Keep::Reg || (L.fr2 && s.dx == 0 && s.dy == 0))) continue;
            for (int iy = 0; iy < L.vy; ++iy)
                for (int jx = 0; jx < L.vx; ++jx) {
                    int c = G.lead + s.dz;
                    const int y = iy + s.dy, x = jx + s.dx;
                    PosInfo &pi = pos[PosKey{s.stage, s.idx, y, x, zqueued(L, s.stage, y, x) ? 0 : c}];
                    pi.cmin = std::min(pi.cmin, c);
                    pi.cmax = std::max(pi.cmax, c);
                }
        }
    return pos;
}

// Region-vector ("frame") evaluation of a statement: its region rows [y_lo, y_lo+rows)
// and x-vector columns [x_lo, x_lo + cs*VW) relative to the tile (x rounded out to the
// 16-byte layout alignment), enumerated as units q = tid + b*NT, q < nq
struct FrameGeo { int x_lo, cs, y_lo, rows, nq, nb; };
static FrameGeo frame_geo(const Launch &L, const Stage &G, int VW) {
    FrameGeo f;
    f.x_lo = -(int)((G.ex0 + VW - 1) / VW * VW);
    const int x_hi = L.tx + (G.ex1 + VW - 1) / VW * VW;
    f.cs = (x_hi - f.x_lo) / VW;
    f.y_lo = -G.ey0;
    f.rows = L.ty + G.ey0 + G.ey1;
    f.nq = f.rows * f.cs;
    f.nb = (f.nq + L.nt - 1) / L.nt;
    return f;
}

// frame mode 2: one unit grid for the whole launch, the union of the statements' regions
static FrameGeo launch_frame(const Launch &L, int VW) {
    int x0 = 0, x1 = L.tx, y0 = 0, y1 = L.ty;
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        const FrameGeo f = frame_geo(L, G, VW);
        x0 = std::min(x0, f.x_lo);
        x1 = std::max(x1, f.x_lo + f.cs * VW);
        y0 = std::min(y0, f.y_lo);
        y1 = std::max(y1, f.y_lo + f.rows);
    }
    FrameGeo f;
    f.x_lo = x0;
    f.cs = (x1 - x0) / VW;
    f.y_lo = y0;
    f.rows = y1 - y0;
    f.nq = f.rows * f.cs;
    f.nb = (f.nq + L.nt - 1) / L.nt;
    return f;
}
// a stage keeps a register queue of its own-position values: register stages always,
// shared-memory stages too in frame mode 2 (their centre / vertical taps)
static bool has_rq(const Launch &L, const Stage &G) {
    return G.keep == Keep::Reg || (L.fr2 && G.keep == Keep::Smem);
}

// registers the generated code keeps live (chooser's occupancy model)
int codegen_regs(const stencil_program *p, const Launch &L) {
    const int w = p->elem / 4;
    int persistent = 0, transient = 0;
    if (L.fr) {
        const int VW = 16 / p->elem;
        for (const Stage &G : L.st) {
            if (!G.needed) continue;
            auto pos = block_positions(L, G);
            const FrameGeo f = L.fr2 ? launch_frame(L, VW) : frame_geo(L, G, VW);
            transient = std::max(transient, ((int)pos.size() + VW) * w * std::min(f.nb, 2));
            if (has_rq(L, G)) persistent += VW * f.nb * G.depth * w;
        }
        if (L.fr2) {  // step-wide input queues of the own-position columns
            const FrameGeo F = launch_frame(L, VW);
            std::map<int, std::pair<int, int>> rng;
            for (const Stage &G : L.st) {
                if (!G.needed) continue;
                for (auto &kv : block_positions(L, G))
                    if (!kv.first.stage && kv.first.y == 0 && kv.first.x == 0) {
                        auto it = rng.emplace(kv.first.id, std::make_pair(kv.second.cmin, kv.second.cmax)).first;
                        it->second.first = std::min(it->second.first, kv.second.cmin);
                        it->second.second = std::max(it->second.second, kv.second.cmax);
                    }
            }
            for (auto &kv : rng)
                if (kv.second.second > kv.second.first)
                    persistent += VW * F.nb * (kv.second.second - kv.second.first + 1) * w;
        }
        return 40 + persistent + transient + 2 * (int)L.in.size();
    }
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        auto pos = block_positions(L, G);
        int direct = 0;
        for (auto &kv : pos) {
            int d = kv.second.cmax - kv.second.cmin + 1;
            if (d > 1) persistent += d * L.cby * w;
            else direct++;
        }
        transient = std::max(transient, (direct + L.vx * L.vy) * w);
        if (G.keep == Keep::Reg) persistent += L.vx * L.vy * L.cby * G.depth * w;
    }
    int halo = 0;
    for (const RegionClass &R : L.cls) {
        int nh = (L.tx + R.x1 - R.x0) * (L.ty + R.y1 - R.y0) - L.tx * L.ty;
        halo += (nh + L.nt - 1) / L.nt * 6;
    }
    return 48 + persistent + transient + halo + 2 * (int)L.in.size();
}

// shared-memory loads per core point over all statements (z-queue refills count
// once per step; direct loads once per block position).  Without z-queues the same
// (layout, y, x, plane) read by several statements of a step is one load: the
// generated loads are plain (non-volatile) and ptxas merges them (checked in SASS).
double codegen_smem_loads(const Launch &L) {
    double loads = 0;
    std::set<PosKey> all;
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        auto pos = block_positions(L, G);
        if (L.zq == 1) loads += (double)pos.size() / (L.vx * L.vy);
        else
            for (auto &kv : pos) all.insert(kv.first);
    }
    return loads + (double)all.size() / (L.vx * L.vy);
}

std::string generate_launch(const stencil_program *p, Launch &L, int index, bool fused) {
    const bool f32 = p->elem == 4;
    const char *T = f32 ? "float" : "double";
    const char *T2 = f32 ? "float4" : "double2";  // 16-byte vector
    const int VW = 16 / p->elem;                   // elements per vector
    const sp_grid &g = p->grid;
    const sp_layout &lay = p->layout;
    const bool tma = p->opt.loader == 0;
    std::ostringstream o;
    L.fn = std::string(fused ? "sf_fused_" : "sf_unfused_") + num(index);
    L.nvtx = L.fn + " " + L.name;
    L.nth = L.nt + (tma ? 32 : 0);
    int XT, YT;
    core_geometry(L, &XT, &YT);
    const int VX = L.vx, VY = L.vy, CBY = L.cby, NPB = VX * VY;
    const bool FR = L.fr;  // region-vector evaluation (frame mode)
    const bool FR2 = FR && L.fr2;  // ... with one unit grid and register z-reuse
    const FrameGeo FF = FR ? launch_frame(L, VW) : FrameGeo{};
    if (FR && (VX != VW || VY != 1 || CBY != 1 || L.tx % VW))
        fail(SP_E_RESOURCES, "internal: frame mode needs 16-byte x-vectors");
    if (!FR && (YT * VY * CBY != L.ty || XT * VX != L.tx || XT * YT != L.nt))
        fail(SP_E_RESOURCES, "internal: inconsistent block geometry");
    for (const RegionClass &R : L.cls)
        if (R.x0 > 0 || R.x1 < 0 || R.y0 > 0 || R.y1 < 0)
            fail(SP_E_RESOURCES, "internal: region class does not contain the tile");

    // pointer slots: arrays whose pointer the kernel needs (stores, ghost loads, LDG loader)
    L.arr_slot.assign(p->arrays.size(), -1);
    L.slot_arr.clear();
    auto need_ptr = [&](int arr) {
        if (L.arr_slot[arr] < 0) {
            L.arr_slot[arr] = (int)L.slot_arr.size();
            L.slot_arr.push_back(arr);
        }
    };
    for (const Stage &G : L.st)
        if (G.needed) need_ptr(G.out);
    if (!tma)
        for (const Input &I : L.in) need_ptr(I.arr);
    const int nin = (int)L.in.size();
    const int narr = (int)L.slot_arr.size();
    L.ptr_off = 128 * (size_t)std::max(nin, 1);
    L.int_off = L.ptr_off + 8 * (size_t)std::max(narr, 1);
    L.xp_off = L.int_off + 24;
    const int NPU = (int)L.pushes.size();
    L.param_size = (L.xp_off + (L.xp ? 40 + 16 * (size_t)std::max(NPU, 1) : 0) + 63) / 64 * 64;
    const int NB = L.nbar_full, NE = L.nbar_empty;
    // thread-block clusters along x (option cluster_x): x-halo values of shared-memory
    // stages inside the neighbouring tile are read from that CTA's ring over DSMEM
    // instead of recomputed; needs whole clusters (ntx % CX == 0), the TMA loader and
    // a shared-memory stage with an x-extension
    {
        int cx = std::max(1, std::min(8, p->opt.cluster_x));
        bool any_x = false;
        for (const Stage &G : L.st)
            if (G.needed && G.keep == Keep::Smem && (G.ex0 > 0 || G.ex1 > 0)) any_x = true;
        if (cx > 1 && (!tma || L.xp || !any_x || L.ntx % cx != 0)) cx = 1;
        L.cx = cx;
    }
    const int CX = L.cx;
    std::vector<int> ready_of(L.st.size(), -1);  // ready mbarrier of a shared x-halo stage
    int n_ready = 0;
    if (CX > 1)
        for (size_t m = 0; m < L.st.size(); ++m) {
            const Stage &G = L.st[m];
            if (G.needed && G.keep == Keep::Smem && (G.ex0 > 0 || G.ex1 > 0)) ready_of[m] = n_ready++;
        }

    o << "// generated by stencilfuse codegen: " << (fused ? "fused group " : "original kernel ")
      << L.name << "\n#define SF_SUSPEND_HINT " << p->opt.suspend_hint
      << "\n#include \"sf_device.cuh\"\n";
    o << "namespace " << L.fn << "_ns {\n";
    o << "typedef " << T << " T;\ntypedef " << T2 << " T2;\n";
    o << "constexpr int TX = " << L.tx << ", TY = " << L.ty << ", NT = " << L.nt << ", ZC = " << L.zc
      << ", KF = " << L.kfirst << ", PF = " << L.pf << ";\n";
    o << "constexpr int CX = " << CX << ";  // CTAs per cluster along x (DSMEM x-halo sharing)\n";
    o << "constexpr int XT = " << XT << ", YT = " << YT << ", VX = " << VX << ", VY = " << VY
      << ", CBY = " << CBY << ";  // thread (xt,yt) owns CBY blocks of VX x VY core points\n";
    o << "constexpr int NX = " << g.nx << ", NY = " << g.ny << ", NZ = " << g.nz_local
      << ", ZLO = " << p->zint_lo << ", ZHI = " << p->zint_hi << ";\n";
    o << "constexpr int XP = " << lay.x_pitch << ", YA = " << lay.y_alloc << ", ZA = " << lay.z_alloc
      << ";\nconstexpr long long PLANE = " << p->plane << ";\n";
    o << "constexpr int OXA = " << lay.origin_x << ", OYA = " << lay.origin_y
      << ", OZA = " << lay.origin_z << ";\n";
    o << "struct __align__(64) Params { SfTmap tm[" << std::max(nin, 1) << "]; T *arr["
      << std::max(narr, 1) << "]; int n_lo, z_mid, z_hi, z_base, z_end, pad_;";
    if (L.xp)  // peer-push protocol: own signal block, neighbours' blocks, peer buffers
        o << "\n  unsigned long long *xs_self, *xs_own, *xs_dn, *xs_up; unsigned *xs_ctr; T *xp["
          << std::max(NPU, 1) << "][2];";
    o << " };\n";
    o << "static_assert(sizeof(SfTmap) * " << std::max(nin, 1) << " == " << L.ptr_off
      << ", \"param layout\");\n";
    // statement coefficients live in constant memory: FP64 FMA/MUL take them as
    // constant-bank operands instead of re-materialising each one per use
    o << "/*SF_COEF_TABLE*/\n}\n";
    // fp64 coefficients are uniform-register operands of DFMA/DMUL on sm_100 (no constant-bank
    // operand); fp32 literals are FFMA immediates, so the table only serves fp64
    const int coef_mode = f32 ? 0 : p->opt.coef_const;
    const bool cc2 = coef_mode == 2;
    std::map<uint64_t, int> coef_idx;
    std::vector<double> coefs;
    auto coef_ref = [&](double c) {
        uint64_t bits;
        std::memcpy(&bits, &c, 8);
        auto it = coef_idx.find(bits);
        if (it == coef_idx.end()) {
            it = coef_idx.emplace(bits, (int)coefs.size()).first;
            coefs.push_back(c);
        }
        // coef_const 2: the index carries a per-step zero read from constant memory, so the
        // address is not loop-invariant: ptxas loads each coefficient right before its use
        // (one LDCU.64 into a uniform register pair) instead of hoisting the whole table into
        // registers (spills) or materialising each literal with two UMOVs (measured in SASS)
        return "SFK[" + num(it->second) + (cc2 ? " + sfz" : "") + "]";
    };
    o << "extern \"C\" __global__ void __launch_bounds__(" << L.nth << ", " << std::max(1, p->opt.minblocks)
      << ") " << L.fn
      << "(const __grid_constant__ " << L.fn << "_ns::Params p) {\n";
    o << "  using namespace " << L.fn << "_ns;\n";
    o << "  extern __shared__ __align__(128) unsigned char sf_smem[];\n";
    o << "  const int tid = threadIdx.x;\n";
    // chunks [0, n_lo) tile planes [z_base, z_mid), the others [z_hi, z_end)
    if (L.xp && L.xp_dw > 0)  // the slab's end chunks go first (order 0, last, 1, 2, ...): they
                              // carry the neighbour exchange, and signal it as soon as done
        o << "  const int bz = sf_xs_chunk((int)blockIdx.z, (int)gridDim.z), lo = bz < p.n_lo;\n";
    else
        o << "  const int bz = (int)blockIdx.z, lo = bz < p.n_lo;\n";
    o << "  const int X0 = (int)blockIdx.x * TX, Y0 = (int)blockIdx.y * TY,\n"
         "            Z0 = lo ? p.z_base + bz * ZC : p.z_hi + (bz - p.n_lo) * ZC;\n";
    o << "  const int zc = min(ZC, (lo ? p.z_mid : p.z_end) - Z0);\n";
    o << "  sf_u64 *full = (sf_u64 *)(sf_smem + " << L.bar_off << ");\n";
    if (tma) o << "  sf_u64 *empty = full + " << NB << ";\n";
    if (CX > 1)
        o << "  const unsigned crank = sf_cluster_rank();\n  sf_u64 *const cready = (sf_u64 *)(sf_smem + "
          << L.ready_off << ");\n";
    for (int a = 0; a < nin; ++a) {
        const Input &I = L.in[a];
        o << "  T *const in" << a << " = (T *)(sf_smem + " << L.in_off[a] << ");  // "
          << p->arrays[I.arr].name << ": " << L.in_rw[a] << "x" << L.in_rh[a] << " x "
          << L.in_depth[a] << " planes, rows " << -I.ey0 << ".., cols " << -I.bx0
          << "..; planes k+[" << I.alo << "," << I.ahi << "], first " << I.qlo << "\n";
    }
    for (size_t m = 0; m < L.st.size(); ++m) {
        const Stage &G = L.st[m];
        if (G.keep == Keep::Smem)
            o << "  T *const st" << m << " = (T *)(sf_smem + " << L.st_off[m] << ");  // "
              << p->arrays[G.out].name << ": " << L.st_w[m] << "x" << L.st_h[m] << " x "
              << L.st_depth[m] << " planes, cols " << -G.sx0 << "..\n";
    }

    // ------------------------------------------------------------ loads
    auto slot_of = [&](int a, const std::string &q) {
        return "((" + q + " - (" + num(L.in[a].qlo) + ")) % " + num(L.in_depth[a]) + ")";
    };
    auto box_bytes = [&](int a) { return (int64_t)L.in_rw[a] * L.in_rh[a] * p->elem; };
    auto issue_plane = [&](int a) {  // plane q of input a (variables q, bar in scope)
        const Input &I = L.in[a];
        std::ostringstream s;
        if (tma) {
            s << "sf_tma_load_3d(in" << a << " + " << slot_of(a, "q") << " * " << L.in_plane[a]
              << ", &p.tm[" << a << "], bar, X0 + (" << -I.bx0 << ") + OXA, Y0 + (" << -I.ey0
              << ") + OYA, Z0 + q + OZA);";
        } else {
            const int rw = L.in_rw[a], rh = L.in_rh[a];
            s << "{ T *dst = in" << a << " + " << slot_of(a, "q") << " * " << L.in_plane[a]
              << "; const int az = Z0 + q + OZA; const T *src = p.arr[" << L.arr_slot[I.arr]
              << "]; for (int e = tid; e < " << rw * rh << "; e += NT) { const int yy = e / " << rw
              << ", xx = e % " << rw << "; const int ax = X0 + (" << -I.bx0
              << ") + OXA + xx, ay = Y0 + (" << -I.ey0 << ") + OYA + yy; "
              << "dst[e] = (ax >= 0 && ax < XP && ay >= 0 && ay < YA && az >= 0 && az < ZA) ? "
              << "src[((long long)az * YA + ay) * XP + ax] : T(0); } }";
        }
        return s.str();
    };
    // batch j: every input's plane j+ahi (and, for j == KF, all earlier planes from qlo);
    // planes below an input's first needed plane qlo are never loaded
    auto q0_of = [&](const Input &I) {
        return "(j == KF) ? " + num(I.qlo) + " : max(j + (" + num(I.ahi) + "), " + num(I.qlo) + ")";
    };
    auto batch = [&](std::ostringstream &s, const std::string &ind) {
        if (tma) {
            s << ind << "unsigned bytes = 0;\n";
            for (int a = 0; a < nin; ++a) {
                const Input &I = L.in[a];
                s << ind << "{ const int q0 = " << q0_of(I) << "; const int q1 = min(j + (" << I.ahi
                  << "), zc - 1 + (" << I.ahi << ")); if (q1 >= q0) bytes += (unsigned)(q1 - q0 + 1) * "
                  << box_bytes(a) << "u; }\n";
            }
            s << ind << "sf_u64 *bar = &full[(j - KF) & " << NB - 1 << "];\n";
            s << ind << "sf_mbar_expect_tx(bar, bytes);\n";
        }
        for (int a = 0; a < nin; ++a) {
            const Input &I = L.in[a];
            s << ind << "{ const int q0 = " << q0_of(I) << "; const int q1 = min(j + (" << I.ahi
              << "), zc - 1 + (" << I.ahi << ")); for (int q = q0; q <= q1; ++q) " << issue_plane(a)
              << " }\n";
        }
    };

    o << "  if (tid == 0) {\n";
    if (tma) {
        o << "    for (int b = 0; b < " << NB << "; ++b) sf_mbar_init(&full[b], 1);\n";
        o << "    for (int b = 0; b < " << NE << "; ++b) sf_mbar_init(&empty[b], " << L.nt / 32
          << ");\n";
        if (n_ready)  // arrivals: every thread of each cluster neighbour, once per plane
            o << "    for (int b = 0; b < " << n_ready << "; ++b) sf_mbar_init(&cready[b], NT * ((crank > 0) + (crank < CX - 1)));\n";
        o << "    sf_fence_mbar_init();\n";
        for (int a = 0; a < nin; ++a) o << "    sf_prefetch_tmap(&p.tm[" << a << "]);\n";
    }
    o << "  }\n  __syncthreads();\n";
    if (CX > 1)  // the neighbours' barriers are initialised before any remote arrival
        o << "  sf_cluster_sync();\n";
    if (L.xp) {
        // peer-push protocol: this kernel is number seq of
        // the rank's launches; a chunk within xp_dw planes of the bottom (top) slab end
        // reads ghost planes the lower (upper) neighbour pushes, or pushes into its
        // ghosts, so it first waits until that neighbour's end chunks facing this rank
        // have completed launch seq-1 (RAW: their pushes are visible; WAR: they have
        // finished reading the ghosts this launch overwrites)
        o << "  sf_pdl_wait();\n";
        // only thread 0 waits and publishes: one load of the counter per CTA (every
        // thread loading the same word would serialise on one L2 slice)
        o << "  const unsigned long long xs_seq = tid == 0 ? sf_ld_volatile_u64(p.xs_self) + 1 : 0;\n";
        if (std::getenv("SF_DEBUG_XP"))  // dev aid (tools/debug_xpush.py): per-CTA trace
            o << "  if (tid == 0) printf(\"[" << L.fn << "] own=%p seq=%llu Z0=%d zc=%d nlo=%d blk=%d,%d,%d\\n\", p.xs_own, xs_seq, Z0, zc, p.n_lo, blockIdx.x, blockIdx.y, blockIdx.z);\n";
        const int DW = L.xp_dw;
        o << "  const bool xs_bot = Z0 < " << DW << ", xs_top = Z0 + zc > NZ - " << DW << ";\n";
        if (DW > 0) {
            o << "  if (xs_bot || xs_top) {\n";
            o << "    if (tid == 0) sf_xs_wait(p.xs_own, xs_bot && p.xs_dn, xs_top && p.xs_up, xs_seq - 1);\n";
            o << "    __syncthreads();\n  }\n";
        }
    }
    // PDL measured r1: -1.6 % on the fused C4 step, +37 % on the 40-launch unfused step
    // (dependent grids parked on griddepcontrol.wait): fused groups only unless pdl=2
    const bool pdl = fused ? p->opt.pdl >= 1 : p->opt.pdl >= 2;
    L.pdl = pdl;
    if (pdl) o << "  sf_pdl_launch_dependents();  // the next group may start its prologue\n";
    if (tma) {
        // the role test uses a warp-uniform value (a shuffle broadcast of the warp index): with
        // a per-thread test ptxas treats the compute loop as possibly divergent and keeps
        // uniform values (the step index, the coefficient-table loads) out of the uniform
        // datapath (micro-kernels: LDC into general registers instead of LDCU)
        o << "  if (__shfl_sync(0xffffffffu, tid >> 5, 0) >= NT / 32) {  // ---- TMA producer warp: batch j for step j, PF steps ahead\n";
        // pbar: the whole producer warp runs the loop and blocks in bar.sync on the step's
        // named barrier until every compute warp has arrived (hardware wait, no polling); one
        // elected lane issues the TMA work.  Named barrier ids 2 .. 2+NE-1 (id 1: compute sync)
        const bool PB = p->opt.pbar && CX == 1 && !L.xp && NE <= 8;
        L.pbar = PB;
        o << (PB ? "    const bool lead = tid == NT;\n    {\n" : "    if (tid == NT) {\n");
        if (pdl) o << "      sf_pdl_wait();  // inputs written by the previous group are complete\n";
        const int L2PF = p->opt.l2pf;
        auto l2_prefetch = [&](const std::string &jexpr, const std::string &ind) {
            // the plane batch `jexpr` will load, prefetched into L2 (independent of the ring)
            for (int a = 0; a < nin; ++a) {
                const Input &I = L.in[a];
                o << ind << "{ const int q = " << jexpr << " + (" << I.ahi << "); if (q >= " << I.qlo
                  << " && q <= zc - 1 + (" << I.ahi << ")) sf_tma_prefetch_3d(&p.tm[" << a
                  << "], X0 + (" << -I.bx0 << ") + OXA, Y0 + (" << -I.ey0
                  << ") + OYA, Z0 + q + OZA); }\n";
            }
        };
        if (L2PF > 0) {
            o << "      " << (PB ? "if (lead) " : "") << "for (int j = KF + 1; j < min(KF + " << L2PF << ", zc); ++j) {\n";
            l2_prefetch("j", "        ");
            o << "      }\n";
        }
        o << "      for (int j = KF; j < zc; ++j) {\n";
        if (L2PF > 0) {
            if (PB) o << "        if (lead) {\n";
            l2_prefetch("(j + " + num(L2PF) + ")", "        ");
            if (PB) o << "        }\n";
        }
        o << "        const int s = j - 1 - PF;  // step whose slots batch j overwrites\n";
        if (PB)
            o << "        if (s >= KF) sf_bar_sync(2 + ((s - KF) & " << NE - 1 << "), NT + 32);\n";
        else if (p->opt.phint > 0)
            o << "        if (s >= KF) sf_mbar_wait_hint(&empty[(s - KF) & " << NE - 1 << "], ((s - KF) >> "
              << log2i(NE) << ") & 1, " << p->opt.phint << "u);\n";
        else if (p->opt.psleep > 0)
            o << "        if (s >= KF) sf_mbar_wait_backoff(&empty[(s - KF) & " << NE - 1 << "], ((s - KF) >> "
              << log2i(NE) << ") & 1, " << p->opt.psleep << "u);\n";
        else
            o << "        if (s >= KF) sf_mbar_wait(&empty[(s - KF) & " << NE - 1 << "], ((s - KF) >> "
              << log2i(NE) << ") & 1);\n";
        if (PB) o << "        if (lead) {\n";
        batch(o, "        ");
        if (PB) o << "        }\n";
        o << "      }\n";
        if (PB)  // the last steps' barrier generations: the compute warps arrive on every step
            o << "      for (int s = max(KF, zc - 1 - PF); s < zc; ++s) sf_bar_sync(2 + ((s - KF) & " << NE - 1
              << "), NT + 32);\n";
        o << "    }\n";
        if (CX > 1) o << "    sf_cluster_sync();  // no CTA leaves while a neighbour may read its rings\n";
        o << "    return;\n  }\n";
    }
    // compute warps store arrays the previous group may still read (WAR) and read
    // what it wrote: wait for its completion before any global access
    if (pdl) o << "  sf_pdl_wait();\n";

    // ---------------------------------------------------- layouts
    struct Lay {
        bool stage;
        int id;
        bool operator<(const Lay &x) const { return std::tie(stage, id) < std::tie(x.stage, x.id); }
    };
    auto lw = [&](const Lay &l) { return l.stage ? L.st_w[l.id] : L.in_rw[l.id]; };
    auto lx0 = [&](const Lay &l) { return l.stage ? -L.st[l.id].sx0 : -L.in[l.id].bx0; };
    auto ly0 = [&](const Lay &l) { return l.stage ? -L.st[l.id].ey0 : -L.in[l.id].ey0; };
    auto lname = [&](const Lay &l) { return std::string(l.stage ? "S" : "I") + num(l.id); };
    std::vector<std::set<Lay>> hlays(L.cls.size());
    std::set<Lay> all_lays;
    for (size_t m = 0; m < L.st.size(); ++m) {
        const Stage &G = L.st[m];
        if (!G.needed) continue;
        if (G.keep == Keep::Smem) {
            hlays[G.cls].insert(Lay{true, (int)m});
            all_lays.insert(Lay{true, (int)m});
        }
        for (const TermR &t : G.terms)
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (s.stage && L.st[s.idx].keep == Keep::Reg) continue;
                hlays[G.cls].insert(Lay{s.stage, s.idx});
                all_lays.insert(Lay{s.stage, s.idx});
            }
    }

    // ---------------------------------------------------- per-thread core tables
    o << "  const int xt = tid % XT, yt = tid / XT;\n";
    o << "  // core block b origin: (xt*VX, (b*YT + yt)*VY); index of its (0,0) in each layout\n";
    for (const Lay &l : all_lays)
        o << "  const int cb_" << lname(l) << " = (yt * VY - (" << ly0(l) << ")) * " << lw(l)
          << " + (xt * VX - (" << lx0(l) << "));\n";
    o << "  const int cg = (Y0 + yt * VY + OYA) * XP + X0 + xt * VX + OXA;\n";
    if (FR) {  // frame mode: every statement's (vector-rounded) region is interior
        int mx0 = 0, mx1 = 0, my0 = 0, my1 = 0;
        for (const Stage &G : L.st) {
            if (!G.needed) continue;
            const FrameGeo f = frame_geo(L, G, VW);
            mx0 = std::max(mx0, -f.x_lo);
            mx1 = std::max(mx1, f.x_lo + f.cs * VW - L.tx);
            my0 = std::max(my0, -f.y_lo);
            my1 = std::max(my1, f.y_lo + f.rows - L.ty);
        }
        o << "  const bool tile_in = X0 >= " << mx0 << " && X0 + TX + " << mx1 << " <= NX && Y0 >= " << my0
          << " && Y0 + TY + " << my1 << " <= NY;  // all regions interior\n";
    } else {
        o << "  const bool tile_in = X0 + TX <= NX && Y0 + TY <= NY;  // all core points interior\n";
    }

    // statement loop bounds (reading R2'): local-coordinate box of a boxed stage
    std::set<int> box_cls;
    auto sbox = [&](const Stage &G, int d) {
        const Stmt &S = p->stmts[G.gid];
        return d >= 4 ? S.box[d] - g.z_offset : S.box[d];
    };
    for (const Stage &G : L.st)
        if (G.needed && p->stmts[G.gid].boxed) box_cls.insert(G.cls);
    // halo tables per class
    std::vector<int> nh(L.cls.size()), hp(L.cls.size());
    for (size_t c = 0; c < L.cls.size(); ++c) {
        if (FR) {  // every region is covered by x-vectors: no point-wise halo strips
            nh[c] = hp[c] = 0;
            continue;
        }
        const RegionClass &R = L.cls[c];
        const int W = L.tx + R.x1 - R.x0, H = L.ty + R.y1 - R.y0;
        nh[c] = W * H - L.tx * L.ty;
        hp[c] = (nh[c] + L.nt - 1) / L.nt;
        o << "  // class " << c << ": x [" << R.x0 << ", TX+" << R.x1 << "), y [" << R.y0 << ", TY+"
          << R.y1 << "), " << W << "x" << H << ": halo " << nh[c] << " points (" << hp[c]
          << " per thread)\n";
        if (!nh[c]) continue;
        o << "  int h" << c << "_f[" << hp[c] << "], h" << c << "_g[" << hp[c] << "];\n";
        if (box_cls.count((int)c))
            o << "  int h" << c << "_x[" << hp[c] << "], h" << c << "_y[" << hp[c] << "];\n";
        for (const Lay &l : hlays[c]) o << "  int h" << c << "_" << lname(l) << "[" << hp[c] << "];\n";
        const int top = -R.y0, bot = R.y1, left = -R.x0, right = R.x1;
        o << "  #pragma unroll\n  for (int i = 0; i < " << hp[c] << "; ++i) {\n";
        o << "    int e = min(tid + i * NT, " << nh[c] - 1 << "), x, y;\n";
        o << "    if (e < " << top * W << ") { y = " << R.y0 << " + e / " << W << "; x = " << R.x0
          << " + e % " << W << "; }\n";
        o << "    else if ((e -= " << top * W << ") < " << bot * W << ") { y = TY + e / " << W
          << "; x = " << R.x0 << " + e % " << W << "; }\n";
        o << "    else { e -= " << bot * W << "; y = e / " << std::max(left + right, 1)
          << "; x = e % " << std::max(left + right, 1) << "; x = x < " << left << " ? x - " << left
          << " : TX + x - " << left << "; }\n";
        o << "    const int gx = X0 + x, gy = Y0 + y, ax = gx + OXA, ay = gy + OYA;\n";
        o << "    h" << c << "_f[i] = ((gx >= 0 && gx < NX && gy >= 0 && gy < NY) ? 2 : 0)"
          << " | ((ax >= 0 && ax < XP && ay >= 0 && ay < YA) ? 8 : 0)";
        if (CX > 1)  // inside the left (16) / right (32) cluster neighbour's tile
            o << " | ((x < 0 && crank > 0) ? 16 : 0) | ((x >= TX && crank < CX - 1) ? 32 : 0)";
        o << ";\n";
        o << "    h" << c << "_g[i] = ay * XP + ax;\n";
        if (box_cls.count((int)c)) o << "    h" << c << "_x[i] = gx; h" << c << "_y[i] = gy;\n";
        for (const Lay &l : hlays[c])
            o << "    h" << c << "_" << lname(l) << "[i] = (y - (" << ly0(l) << ")) * " << lw(l)
              << " + (x - (" << lx0(l) << "));\n";
        o << "  }\n";
    }

    // register stages (core blocks + halo points) and z-queues of block positions
    std::vector<std::map<PosKey, PosInfo>> bpos(L.st.size());
    for (size_t m = 0; m < L.st.size(); ++m) {
        const Stage &G = L.st[m];
        if (!G.needed) continue;
        bpos[m] = block_positions(L, G);
        if (has_rq(L, G)) {
            o << "  T rq" << m << "[" << (FR2 ? FF.nb : FR ? frame_geo(L, G, VW).nb : CBY) << "][" << NPB << "]["
              << G.depth << "];\n";
            if (nh[G.cls]) o << "  T rh" << m << "[" << hp[G.cls] << "][" << G.depth << "];\n";
        }
    }
    auto qname = [&](int m, const PosKey &k) {
        return "zq" + num(m) + "_" + (k.stage ? "S" : "I") + num(k.id) + "_" + sg(k.y) + "_" + sg(k.x);
    };
    // zq 2: step-wide input queues (union of the plane ranges of all statements)
    std::map<PosKey, PosInfo> gq;
    if (L.zq == 2) {
        for (size_t m = 0; m < L.st.size(); ++m)
            for (auto &kv : bpos[m])
                if (!kv.first.stage && zqueued(L, false, kv.first.y, kv.first.x)) {
                    PosInfo &g = gq[kv.first];
                    g.cmin = std::min(g.cmin, kv.second.cmin);
                    g.cmax = std::max(g.cmax, kv.second.cmax);
                }
        for (auto it = gq.begin(); it != gq.end();)
            it = it->second.cmax > it->second.cmin ? std::next(it) : gq.erase(it);
        if (FR2) {
            // frame mode 2 refills a unit's whole x-vector per plane: every lane of an input
            // with a queued lane gets the union plane range (taps with dx != 0 reach some
            // lanes of the own vector, so lanes differ in the planes they are read at)
            std::map<int, PosInfo> un;
            for (auto &kv : gq) {
                PosInfo &u = un[kv.first.id];
                u.cmin = std::min(u.cmin, kv.second.cmin);
                u.cmax = std::max(u.cmax, kv.second.cmax);
            }
            gq.clear();
            for (auto &kv : un)
                for (int x = 0; x < VW; ++x) gq[PosKey{false, kv.first, 0, x, 0}] = kv.second;
        }
    }
    auto gqname = [&](const PosKey &k) {
        return "zg_I" + num(k.id) + "_" + sg(k.y) + "_" + sg(k.x);
    };
    for (auto &kv : gq)
        o << "  T " << gqname(kv.first) << "[" << (FR2 ? num(FF.nb) : "CBY") << "]["
          << kv.second.cmax - kv.second.cmin + 1 << "];\n";
    if (L.zq == 1)
        for (size_t m = 0; m < L.st.size(); ++m)
            for (auto &kv : bpos[m])
                if (kv.second.cmax > kv.second.cmin)
                    o << "  T " << qname((int)m, kv.first) << "[CBY][" << kv.second.cmax - kv.second.cmin + 1
                      << "];\n";
    if (!tma) {
        o << "  for (int j = KF; j < min(KF + PF, zc); ++j) {\n";
        batch(o, "    ");
        o << "  }\n  sf_bar_sync(1, NT);\n";
    }

    // ------------------------------------------------------------- z-march
    for (int r = 0; r < n_ready; ++r) o << "  unsigned cph" << r << " = 0;\n";
    // coef_const 2: a toggle used only to index the zero table keeps the coefficient address
    // warp-uniform in ptxas's analysis (the step index itself feeds per-thread addressing and
    // lives in a general register), so each coefficient is one LDCU into a uniform register
    if (cc2) o << "  unsigned sfc = 0u;\n";
    o << "  for (int k = KF; k < zc; ++k) {\n";
    if (cc2) o << "    sfc ^= 1u;\n    const int sfz = SFZ[sfc];  // always 0 (see coef_ref)\n";
    if (tma) {
        o << "    sf_mbar_wait(&full[(k - KF) & " << NB - 1 << "], ((k - KF) >> " << log2i(NB)
          << ") & 1);\n";
    } else {
        o << "    { const int j = k + PF; if (j < zc) {\n";
        batch(o, "      ");
        o << "    } }\n";
    }
    // per-step plane bases for every (layout, plane offset c relative to k) used
    std::set<std::pair<Lay, int>> basekeys;
    for (size_t m = 0; m < L.st.size(); ++m) {
        const Stage &G = L.st[m];
        if (!G.needed) continue;
        if (G.keep == Keep::Smem) basekeys.insert({Lay{true, (int)m}, G.lead});
        for (const TermR &t : G.terms)
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (s.stage && L.st[s.idx].keep == Keep::Reg) continue;
                basekeys.insert({Lay{s.stage, s.idx}, G.lead + s.dz});
            }
        for (auto &kv : bpos[m])  // queue fills at the first step read every plane offset
            for (int c = kv.second.cmin; c <= kv.second.cmax; ++c)
                basekeys.insert({Lay{kv.first.stage, kv.first.id}, c});
    }
    for (auto &kv : gq)
        for (int c = kv.second.cmin; c <= kv.second.cmax; ++c)
            basekeys.insert({Lay{false, kv.first.id}, c});
    auto bname = [&](const Lay &l, int c) { return "B" + lname(l) + "_" + sg(c); };
    // ring slot of plane k + c in a ring whose slot 0 holds plane lo: (k + c - lo) mod D,
    // shifted by a multiple of D so the operand is non-negative for every step k >= KF
    // (an unsigned modulo: a mask or a multiply-high instead of the signed sequence)
    auto uslot = [&](int c, int lo, int D) {
        const int need = lo - c - L.kfirst;
        const int M = need > 0 ? (need + D - 1) / D : 0;
        return "((unsigned)(k + (" + num(c - lo + D * M) + ")) % " + num(D) + "u)";
    };
    for (auto &bk : basekeys) {
        const Lay &l = bk.first;
        const int c = bk.second;
        std::string slot;
        int64_t plane;
        if (l.stage) {
            slot = uslot(c, L.st[l.id].loff, L.st_depth[l.id]);
            plane = L.st_plane[l.id];
        } else {
            slot = uslot(c, L.in[l.id].qlo, L.in_depth[l.id]);
            plane = L.in_plane[l.id];
        }
        o << "    T *const " << bname(l, c) << " = " << (l.stage ? "st" : "in") << l.id << " + " << slot
          << " * " << plane << ";\n";
    }
    if (!gq.empty() && FR2) {
        // frame mode 2: every thread refills the own-position columns of its units (one
        // 16-byte vector per input and unit: all VW lanes share the plane range) — units
        // outside an input's loaded box keep stale values nobody reads
        std::map<int, std::pair<int, int>> cols;  // input -> plane range of its queues
        for (auto &kv : gq) cols[kv.first.id] = {kv.second.cmin, kv.second.cmax};
        for (auto &kv : gq)
            if (kv.second.cmin != cols[kv.first.id].first || kv.second.cmax != cols[kv.first.id].second)
                fail(SP_E_RESOURCES, "internal: frame-2 input queue lanes differ in plane range");
        o << "    #pragma unroll\n    for (int b = 0; b < " << FF.nb << "; ++b) {\n";
        o << "      const int qq = tid + b * NT;\n";
        o << "      const int fy = " << FF.y_lo << " + qq / " << FF.cs << ", fx = " << FF.x_lo << " + (qq % "
          << FF.cs << ") * " << VW << ";\n";
        for (auto &cv : cols) {
            const int a = cv.first;
            const Input &I = L.in[a];
            Lay l{false, a};
            const int cmin = cv.second.first, cmax = cv.second.second;
            o << "      if (qq < " << FF.nq << " && fy >= " << -I.ey0 << " && fy < TY + " << I.ey1 << " && fx >= "
              << -I.bx0 << " && fx + " << VW << " <= " << -I.bx0 + L.in_rw[a] << ") {\n";
            o << "        const int fi = (fy - (" << ly0(l) << ")) * " << lw(l) << " + (fx - (" << lx0(l) << "));\n";
            auto vload = [&](int cc, const std::string &dst_idx) {
                // one vector of the unit's VW lanes at plane offset cc; planes below the
                // input's first loaded plane are never consumed: do not touch their slots
                o << "          { const T2 v = (k + (" << cc << ") >= (" << I.qlo
                  << ")) ? *reinterpret_cast<const T2 *>(" << bname(l, cc) << " + fi) : T2{};\n";
                const char *comp[4] = {"x", "y", "z", "w"};
                for (int e2 = 0; e2 < VW; ++e2)
                    o << "            " << gqname(PosKey{false, a, 0, e2, 0}) << "[b][" << dst_idx << "] = v."
                      << comp[e2] << ";\n";
                o << "          }\n";
            };
            o << "        if (k == KF) {\n";
            for (int cc = cmin; cc <= cmax; ++cc) vload(cc, num(cc - cmin));
            o << "        } else {\n";
            for (int e2 = 0; e2 < VW; ++e2) {
                const std::string q = gqname(PosKey{false, a, 0, e2, 0});
                for (int d = 0; d < cmax - cmin; ++d)
                    o << "          " << q << "[b][" << d << "] = " << q << "[b][" << d + 1 << "];\n";
            }
            vload(cmax, num(cmax - cmin));
            o << "        }\n      }\n";
        }
        o << "    }\n";
    } else if (!gq.empty()) {
        auto gaddr = [&](const PosKey &k, int cc) {
            Lay l{false, k.id};
            return bname(l, cc) + " + cb_" + lname(l) + " + b * (YT * VY * " + num(lw(l)) + ") + (" +
                   num(k.y * lw(l) + k.x) + ")";
        };
        o << "    #pragma unroll\n    for (int b = 0; b < CBY; ++b) {\n      if (k == KF) {\n";
        // planes below the input's first loaded plane (statements not yet active at
        // the first steps) are never consumed: do not touch their (unloaded) slots
        auto gload = [&](const PosKey &k, int cc) {
            return "(k + (" + num(cc) + ") >= (" + num(L.in[k.id].qlo) + ") ? *(" + gaddr(k, cc) +
                   ") : T(0))";
        };
        for (auto &kv : gq)
            for (int cc = kv.second.cmin; cc <= kv.second.cmax; ++cc)
                o << "        " << gqname(kv.first) << "[b][" << cc - kv.second.cmin << "] = "
                  << gload(kv.first, cc) << ";\n";
        o << "      } else {\n";
        for (auto &kv : gq) {
            const std::string q = gqname(kv.first);
            const int r = kv.second.cmax - kv.second.cmin;
            for (int d = 0; d < r; ++d)
                o << "        " << q << "[b][" << d << "] = " << q << "[b][" << d + 1 << "];\n";
            o << "        " << q << "[b][" << r << "] = " << gload(kv.first, kv.second.cmax) << ";\n";
        }
        o << "      }\n    }\n";
    }

    // Step body, emitted twice when possible: FP (fast step) = an interior tile at a
    // step where every statement's plane lies inside the slab's global interior (and,
    // for stored statements, inside the chunk): every range / ghost / store predicate
    // is then the constant true and the compiler drops those branches; the general
    // body serves edge tiles, warm-up steps and the chunk's last planes.  Both bodies
    // evaluate the same expressions in the same order (bit-identical results).
    bool any_boxed = false;
    for (const Stage &G : L.st)
        if (G.needed && p->stmts[G.gid].boxed) any_boxed = true;
    const int fpmode = L.fastpath >= 0 ? L.fastpath : p->opt.fastpath;
    const bool spec = fpmode != 0 && !any_boxed;
    // fastpath 2: the fast body also runs the chunk's warm-up steps (statements before their
    // first plane compute values nobody reads; stores keep a uniform plane-range test), so
    // only chunks / tiles at the global boundary ever execute the general body — one hot
    // body per CTA instead of two (the instruction cache held both, r2 measurements)
    const bool spec2 = spec && fpmode == 2;
    if (spec) {
        int kst0 = INT32_MIN;
        int lmin = INT32_MAX, lmax = INT32_MIN, slmin = INT32_MAX, slmax = INT32_MIN;
        for (const Stage &G : L.st) {
            if (!G.needed) continue;
            kst0 = std::max(kst0, G.loff - G.lead);
            lmin = std::min(lmin, G.lead);
            lmax = std::max(lmax, G.lead);
            if (G.stored) { slmin = std::min(slmin, G.lead); slmax = std::max(slmax, G.lead); }
        }
        o << "    // fast-step window [sf_k0, sf_k1) of this chunk (see codegen.cpp)\n";
        o << "    int sf_k0 = max(" << (spec2 ? std::string("KF") : num(kst0)) << ", ZLO - Z0 - (" << lmin
          << ")), sf_k1 = min(zc, ZHI - Z0 - (" << lmax << "));\n";
        if (slmin != INT32_MAX && !spec2)
            o << "    sf_k0 = max(sf_k0, -(" << slmin << ")); sf_k1 = min(sf_k1, zc - (" << slmax << "));\n";
    }
    auto emit_body = [&](const bool FP) {
    std::set<int> dirty;
    for (size_t mi = 0; mi < L.st.size(); ++mi) {
        const int m = (int)mi;
        const Stage &G = L.st[m];
        if (!G.needed) continue;
        const Stmt &S = p->stmts[G.gid];
        bool need_bar = G.war_barrier;
        for (const TermR &t : G.terms)
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (s.stage && dirty.count(s.idx)) need_bar = true;
            }
        if (need_bar) {
            o << "    sf_bar_sync(1, NT);\n";
            dirty.clear();
        }
        const int c = G.cls;
        const auto &pos = bpos[m];
        o << "    { // stmt " << p->kernels[S.kernel].name << ":" << S.local << " -> "
          << p->arrays[G.out].name << "  lead " << G.lead << ", planes [" << G.loff << ", zc-1+"
          << G.lead << "], ext (" << G.ex0 << "," << G.ex1 << "," << G.ey0 << "," << G.ey1 << ")"
          << (G.stored ? ", stored" : "") << (G.keep == Keep::Reg ? ", register" : ", smem ring")
          << " depth " << G.depth << "\n";
        // register-stage queues advance every step
        if (has_rq(L, G) && G.depth > 1) {
            o << "      #pragma unroll\n      for (int b = 0; b < " << (FR2 ? num(FF.nb) : FR ? num(frame_geo(L, G, VW).nb) : "CBY")
              << "; ++b)\n"
              << "      #pragma unroll\n      for (int i = 0; i < " << NPB << "; ++i)\n"
              << "      #pragma unroll\n      for (int d = 0; d < " << G.depth - 1 << "; ++d) rq" << m
              << "[b][i][d] = rq" << m << "[b][i][d + 1];\n";
            if (nh[c])
                o << "      #pragma unroll\n      for (int i = 0; i < " << hp[c] << "; ++i)\n"
                  << "      #pragma unroll\n      for (int d = 0; d < " << G.depth - 1 << "; ++d) rh"
                  << m << "[i][d] = rh" << m << "[i][d + 1];\n";
        }
        // address of a block position in a layout at plane offset cc
        auto baddr = [&](const PosKey &k, int cc) {
            Lay l{k.stage, k.id};
            if (FR) return bname(l, cc) + " + fi_" + lname(l) + " + (" + num(k.y * lw(l) + k.x) + ")";
            return bname(l, cc) + " + cb_" + lname(l) + " + b * (YT * VY * " + num(lw(l)) + ") + (" +
                   num(k.y * lw(l) + k.x) + ")";
        };
        // z-queues: advance, refill the newest plane (every step: the pipeline is uniform)
        bool any_q = false;
        if (L.zq == 1)
            for (auto &kv : pos)
                if (kv.second.cmax > kv.second.cmin) any_q = true;
        if (any_q) {
            o << "      #pragma unroll\n      for (int b = 0; b < CBY; ++b) {\n";
            o << "        if (k == KF) {\n";
            for (auto &kv : pos) {
                const PosInfo &pi = kv.second;
                if (pi.cmax == pi.cmin) continue;
                for (int cc = pi.cmin; cc <= pi.cmax; ++cc)
                    o << "          " << qname(m, kv.first) << "[b][" << cc - pi.cmin << "] = *("
                      << baddr(kv.first, cc) << ");\n";
            }
            o << "        } else {\n";
            for (auto &kv : pos) {
                const PosInfo &pi = kv.second;
                if (pi.cmax == pi.cmin) continue;
                const std::string q = qname(m, kv.first);
                for (int d = 0; d < pi.cmax - pi.cmin; ++d)
                    o << "          " << q << "[b][" << d << "] = " << q << "[b][" << d + 1 << "];\n";
                o << "          " << q << "[b][" << pi.cmax - pi.cmin << "] = *("
                  << baddr(kv.first, pi.cmax) << ");\n";
            }
            o << "        }\n      }\n";
        }
        o << "      const int q = k + (" << G.lead << ");\n";
        if (FP) o << "      {\n";
        else o << "      if (q >= (" << G.loff << ") && q <= zc - 1 + (" << G.lead << ")) {\n";
        o << "        const int gz = Z0 + q;\n";
        const bool boxed = p->stmts[G.gid].boxed;
        // in-box tests of this statement (the whole interior unless boxed)
        const std::string BX0 = boxed ? num(sbox(G, 0)) : "0", BX1 = boxed ? num(sbox(G, 1)) : "NX";
        const std::string BY0 = boxed ? num(sbox(G, 2)) : "0", BY1 = boxed ? num(sbox(G, 3)) : "NY";
        if (FP)
            o << "        const bool zin = true;  // fast step\n";
        else if (boxed)
            o << "        const bool zin = gz >= (" << sbox(G, 4) << ") && gz < (" << sbox(G, 5)
              << ");  // loop bounds (R2')\n";
        else
            o << "        const bool zin = gz >= ZLO && gz < ZHI;\n";
        o << "        const bool zal = " << (FP ? "true" : "gz + OZA >= 0 && gz + OZA < ZA") << ";\n";
        o << "        T *const gpl = p.arr[" << L.arr_slot[G.out] << "] + (long long)(gz + OZA) * PLANE;\n";
        if (G.stored)
            o << "        const bool zst = " << (FP && !spec2 ? "true" : "q >= 0 && q < zc") << ";\n";
        if (FP)
            o << "        const bool fast = true;\n";
        else if (boxed)
            o << "        const bool fast = X0 >= " << BX0 << " && X0 + TX <= " << BX1 << " && Y0 >= "
              << BY0 << " && Y0 + TY <= " << BY1 << " && zin;\n";
        else if (FR) {  // the statement's whole (vector-rounded) region is interior
            const FrameGeo f = frame_geo(L, G, VW);
            o << "        const bool fast = zin && X0 + (" << f.x_lo << ") >= 0 && X0 + (" << f.x_lo + f.cs * VW
              << ") <= NX && Y0 + (" << f.y_lo << ") >= 0 && Y0 + (" << f.y_lo + f.rows << ") <= NY;\n";
        } else
            o << "        const bool fast = tile_in && zin;\n";

        // ---- core blocks (frame mode: the region's x-vectors, unit q = tid + b*NT)
        std::string GX0 = "X0 + xt * VX", GY0 = "Y0 + by", GOFF = "cg + b * (YT * VY * XP)";
        std::string blk_close = "        }\n";
        if (FR) {
            const FrameGeo fs = frame_geo(L, G, VW);
            const FrameGeo f = FR2 ? FF : fs;  // enumeration: own region, or the launch frame
            o << "        #pragma unroll\n        for (int b = 0; b < " << f.nb << "; ++b) {\n";
            o << "          const int qq = tid + b * NT;\n";
            o << "          const int fy = " << f.y_lo << " + qq / " << f.cs << ", fx = " << f.x_lo << " + (qq % "
              << f.cs << ") * " << VW << ";\n";
            std::string act;
            if (f.nq % L.nt) act = "qq < " + num(f.nq);
            if (FR2 && (fs.y_lo != FF.y_lo || fs.rows != FF.rows || fs.x_lo != FF.x_lo || fs.cs != FF.cs))
                act += std::string(act.empty() ? "" : " && ") + "fy >= " + num(fs.y_lo) + " && fy < " +
                       num(fs.y_lo + fs.rows) + " && fx >= " + num(fs.x_lo) + " && fx < " +
                       num(fs.x_lo + fs.cs * VW);
            if (!act.empty()) {
                o << "          if (" << act << ") {\n";
                blk_close = "          }\n        }\n";
            }
            std::set<Lay> used;
            if (G.keep == Keep::Smem) used.insert(Lay{true, m});
            for (auto &kv : pos) used.insert(Lay{kv.first.stage, kv.first.id});
            for (const Lay &l : used)
                o << "          const int fi_" << lname(l) << " = (fy - (" << ly0(l) << ")) * " << lw(l)
                  << " + (fx - (" << lx0(l) << "));\n";
            GX0 = "X0 + fx";
            GY0 = "Y0 + fy";
            GOFF = "((Y0 + fy + OYA) * XP + X0 + fx + OXA)";
        } else {
            o << "        #pragma unroll\n        for (int b = 0; b < CBY; ++b) {\n";
        }
        // direct loads, vectorised along x where aligned
        std::map<std::tuple<bool, int, int, int>, std::set<int>> rows;  // (stage,id,c,y) -> xs
        for (auto &kv : pos)
            if (kv.second.cmax == kv.second.cmin && !gq.count(kv.first))
                rows[std::make_tuple(kv.first.stage, kv.first.id, kv.second.cmin, kv.first.y)].insert(
                    kv.first.x);
        auto dname = [&](bool st, int id, int cc, int y, int x) {
            return std::string("d_") + (st ? "S" : "I") + num(id) + "_" + sg(cc) + "_" + sg(y) + "_" +
                   sg(x);
        };
        const bool vec_ok = VW > 1 && VX % VW == 0;
        for (auto &rw : rows) {
            bool st;
            int id, cc, y;
            std::tie(st, id, cc, y) = rw.first;
            const std::set<int> &xs = rw.second;
            std::set<int> done;
            for (int x : xs) {
                if (done.count(x)) continue;
                // 16-byte vector starting at an aligned x (block origins and layouts are aligned)
                int xa = x - (((x % VW) + VW) % VW);
                int cnt = 0;
                for (int e2 = 0; e2 < VW; ++e2) cnt += (int)xs.count(xa + e2);
                if (vec_ok && cnt >= 2) {
                    std::string vn = "v" + dname(st, id, cc, y, xa);
                    o << "          const T2 " << vn << " = *reinterpret_cast<const T2 *>("
                      << baddr(PosKey{st, id, y, xa, 0}, cc) << ");\n";
                    const char *comp[4] = {"x", "y", "z", "w"};
                    for (int e2 = 0; e2 < VW; ++e2)
                        if (xs.count(xa + e2)) {
                            o << "          const T " << dname(st, id, cc, y, xa + e2) << " = " << vn
                              << "." << comp[e2] << ";\n";
                            done.insert(xa + e2);
                        }
                } else {
                    o << "          const T " << dname(st, id, cc, y, x) << " = *("
                      << baddr(PosKey{st, id, y, x, 0}, cc) << ");\n";
                    done.insert(x);
                }
            }
        }
        // expressions of the VX*VY block points
        auto core_operand = [&](const Src &s, int iy, int jx) -> std::string {
            if (s.stage && (L.st[s.idx].keep == Keep::Reg || (FR2 && s.dx == 0 && s.dy == 0))) {
                const Stage &P = L.st[s.idx];
                int d = G.lead + s.dz - P.lead + P.depth - 1;
                return "rq" + num(s.idx) + "[b][" + num(iy * VX + jx) + "][" + num(d) + "]";
            }
            int cc = G.lead + s.dz;
            const int y = iy + s.dy, x = jx + s.dx;
            PosKey k{s.stage, s.idx, y, x, zqueued(L, s.stage, y, x) ? 0 : cc};
            auto g = gq.find(k);
            if (g != gq.end()) return gqname(k) + "[b][" + num(cc - g->second.cmin) + "]";
            const PosInfo &pi = pos.at(k);
            if (pi.cmax > pi.cmin) return qname(m, k) + "[b][" + num(cc - pi.cmin) + "]";
            return dname(s.stage, s.idx, cc, k.y, k.x);
        };
        // Parity build (fmad=0): one left-to-right sum, the fixed order of R4 (bit-exact
        // with the oracle).  Perf build: ACC interleaved partial sums (term t goes to sum
        // t % ACC) added at the end — independent FMA chains for ILP; the reassociation
        // is within the 1e-12 / 1e-5 tolerance like the FMA contraction itself.
        const int ACC = (p->opt.fmad && G.terms.size() >= 6) ? p->opt.acc_split : 1;
        // Perf build, factor=1: the terms sharing one b operand (SCALE-LES-style flux
        // c_t * a[p+o_t] * m[p]) become m * (sum of c_t * a): one multiply per distinct b
        // instead of one per term — exact in real arithmetic, a reassociation within the
        // tolerance like the FMA contraction; the parity build keeps R4's form.
        std::vector<std::vector<int>> items;  // term indices; >1 entries = one shared b
        {
            const bool fac = p->opt.fmad && p->opt.factor;
            for (int ti = 0; ti < (int)G.terms.size(); ++ti) {
                const TermR &t = G.terms[ti];
                bool placed = false;
                if (fac && t.has_b)
                    for (auto &it : items) {
                        const TermR &u = G.terms[it[0]];
                        if (u.has_b && u.b.stage == t.b.stage && u.b.idx == t.b.idx &&
                            u.b.dx == t.b.dx && u.b.dy == t.b.dy && u.b.dz == t.b.dz) {
                            it.push_back(ti);
                            placed = true;
                            break;
                        }
                    }
                if (!placed) items.push_back({ti});
            }
        }
        auto term_expr = [&](const std::function<std::string(const Src &)> &opd) {
            auto scaled = [&](const TermR &t) {
                std::string a = opd(t.a);
                if (t.coef == 1.0) return a;
                if (t.coef == -1.0) return "(-" + a + ")";
                return (coef_mode ? coef_ref(t.coef) : "(T)" + lit(t.coef, f32)) + " * " +
                       a;
            };
            std::vector<std::string> part(ACC);
            for (size_t ii = 0; ii < items.size(); ++ii) {
                const std::vector<int> &it = items[ii];
                std::string term;
                if (it.size() == 1) {
                    const TermR &t = G.terms[it[0]];
                    term = scaled(t);
                    if (t.has_b) term = "(" + term + ") * " + opd(t.b);
                } else {
                    std::string s;
                    for (int ti : it) s = s.empty() ? scaled(G.terms[ti]) : "(" + s + ") + " +
                                                                                scaled(G.terms[ti]);
                    term = "(" + s + ") * " + opd(G.terms[it[0]].b);
                }
                std::string &e = part[ii % ACC];
                e = e.empty() ? term : "(" + e + ") + " + term;
            }
            std::string e = part[0];
            for (int a = 1; a < ACC; ++a)
                if (!part[a].empty()) e = "(" + e + ") + (" + part[a] + ")";
            return e;
        };
        for (int iy = 0; iy < VY; ++iy)
            for (int jx = 0; jx < VX; ++jx)
                o << "          T o" << iy << "_" << jx << " = "
                  << term_expr([&](const Src &s) { return core_operand(s, iy, jx); }) << ";\n";
        // ghost substitution and store predicates outside the interior (edge tiles, z ghosts)
        if (!FR) o << "          const int by = (b * YT + yt) * VY;\n";
        o << "          if (!fast) {\n";
        for (int iy = 0; iy < VY; ++iy)
            for (int jx = 0; jx < VX; ++jx) {
                std::string gx = GX0 + " + " + num(jx), gy = GY0 + " + " + num(iy);
                std::string inb = boxed ? gx + " >= " + BX0 + " && " + gx + " < " + BX1 +
                                              " && " + gy + " >= " + BY0 + " && " + gy + " < " + BY1
                                        : gx + " < NX && " + gy + " < NY";
                std::string alloc = gx + " < XP - OXA && " + gy + " < YA - OYA";
                if (FR) {  // region points left of / above the tile as well
                    inb = gx + " >= 0 && " + gy + " >= 0 && " + inb;
                    alloc = gx + " + OXA >= 0 && " + gy + " + OYA >= 0 && " + alloc;
                }
                o << "            if (!(zin && " << inb << ")) o" << iy << "_"
                  << jx << " = sf_ldg_pred(gpl + " << GOFF << " + (" << iy << " * XP + " << jx
                  << "), zal && " << alloc << ");\n";
            }
        o << "          }\n";
        // sinks
        if (G.keep == Keep::Smem) {
            Lay self{true, m};
            for (int iy = 0; iy < VY; ++iy) {
                std::string a = FR ? bname(self, G.lead) + " + fi_" + lname(self) + " + (" +
                                         num(iy * lw(self)) + ")"
                                   : bname(self, G.lead) + " + cb_" + lname(self) + " + b * (YT * VY * " +
                                         num(lw(self)) + ") + (" + num(iy * lw(self)) + ")";
                if (vec_ok) {
                    for (int jx = 0; jx < VX; jx += VW) {
                        o << "          *reinterpret_cast<T2 *>(" << a << " + " << jx << ") = T2{";
                        for (int e2 = 0; e2 < VW; ++e2)
                            o << (e2 ? ", " : "") << "o" << iy << "_" << jx + e2;
                        o << "};\n";
                    }
                } else {
                    for (int jx = 0; jx < VX; ++jx)
                        o << "          *(" << a << " + " << jx << ") = o" << iy << "_" << jx << ";\n";
                }
            }
        }
        if (has_rq(L, G)) {
            for (int iy = 0; iy < VY; ++iy)
                for (int jx = 0; jx < VX; ++jx)
                    o << "          rq" << m << "[b][" << iy * VX + jx << "][" << G.depth - 1 << "] = o"
                      << iy << "_" << jx << ";\n";
        }
        if (G.stored) {
            // the tile's core points of this plane, stored at base pointer `gbn`
            auto stores = [&](const std::string &gbn, const std::string &ind) {
                o << ind << "if (fast) {\n";
                for (int iy = 0; iy < VY; ++iy) {
                    if (vec_ok) {
                        for (int jx = 0; jx < VX; jx += VW) {
                            o << ind << "  sf_st_v(" << gbn << " + (" << iy << " * XP + " << jx << "), T2{";
                            for (int e2 = 0; e2 < VW; ++e2)
                                o << (e2 ? ", " : "") << "o" << iy << "_" << jx + e2;
                            o << "});\n";
                        }
                    } else {
                        for (int jx = 0; jx < VX; ++jx)
                            o << ind << "  sf_st(" << gbn << " + (" << iy << " * XP + " << jx << "), o" << iy
                              << "_" << jx << ");\n";
                    }
                }
                o << ind << "} else {\n";
                for (int iy = 0; iy < VY; ++iy)
                    for (int jx = 0; jx < VX; ++jx) {
                        const std::string gx = GX0 + " + " + num(jx), gy = GY0 + " + " + num(iy);
                        const std::string inb = boxed ? "zin && " + gx + " >= " + BX0 + " && " + gx + " < " +
                                                            BX1 + " && " + gy + " >= " + BY0 + " && " + gy +
                                                            " < " + BY1
                                                      : gx + " < NX && " + gy + " < NY";
                        o << ind << "  if (" << inb << ") sf_st(" << gbn << " + (" << iy << " * XP + " << jx
                          << "), o" << iy << "_" << jx << ");\n";
                    }
                o << ind << "}\n";
            };
            if (FR)  // frame units inside the tile core (x-vectors are whole: TX % VW == 0)
                o << "          if (zst && fy >= 0 && fy < TY && fx >= 0 && fx < TX) {\n";
            else
                o << "          if (zst) {\n";
            o << "            T *const gb = gpl + " << GOFF << ";\n";
            stores("gb", "            ");
            for (size_t k = 0; k < L.pushes.size(); ++k) {
                const Launch::Push &u = L.pushes[k];
                if (u.stage != (int)m) continue;
                // the same element of the neighbour's buffer, one slab up/down (layouts are
                // identical on every rank): its top / bottom ghost planes
                const std::string off = "(gb - p.arr[" + num(L.arr_slot[G.out]) + "])";
                if (u.dn > 0) {
                    o << "            if (gz < " << u.dn << " && p.xp[" << k << "][0]) {  // push down\n";
                    o << "              T *const pb = p.xp[" << k << "][0] + " << off << " + (long long)NZ * PLANE;\n";
                    stores("pb", "              ");
                    o << "            }\n";
                }
                if (u.up > 0) {
                    o << "            if (gz >= NZ - " << u.up << " && p.xp[" << k << "][1]) {  // push up\n";
                    o << "              T *const pb = p.xp[" << k << "][1] + " << off << " - (long long)NZ * PLANE;\n";
                    stores("pb", "              ");
                    o << "            }\n";
                }
            }
            o << "          }\n";
        }
        o << blk_close;

        // ---- halo points (point-wise)
        if (nh[c]) {
            auto halo_operand = [&](const Src &s) -> std::string {
                if (s.stage && L.st[s.idx].keep == Keep::Reg) {
                    const Stage &P = L.st[s.idx];
                    int d = G.lead + s.dz - P.lead + P.depth - 1;
                    return "rh" + num(s.idx) + "[i][" + num(d) + "]";
                }
                Lay l{s.stage, s.idx};
                int off = s.dy * lw(l) + s.dx;
                return bname(l, G.lead + s.dz) + "[h" + num(c) + "_" + lname(l) + "[i] + (" +
                       num(off) + ")]";
            };
            o << "        #pragma unroll\n        for (int i = 0; i < " << hp[c] << "; ++i) {\n";
            o << "          const int f = h" << c << "_f[i];\n";
            if (CX > 1) o << "          if (f & 48) continue;  // the cluster neighbour computes it\n";
            // ghost points (e.g. the y-halo rows of full-height tiles) are only loaded
            std::string hin;  // the point is evaluated (not a ghost / outside the loop box)
            if (boxed) {
                o << "          const int hx = h" << c << "_x[i], hy = h" << c << "_y[i];\n";
                hin = "zin && hx >= " + BX0 + " && hx < " + BX1 + " && hy >= " + BY0 + " && hy < " + BY1;
            } else {
                hin = "zin && (f & 2)";
            }
            if (p->opt.halo_sel) {
                // every halo point's expression is evaluated (its operands are inside the
                // layouts; a ghost point's value is discarded) and the ghost value replaces
                // it after: no branch around the loads, so the unrolled points interleave
                o << "          T v = " << term_expr(halo_operand) << ";\n";
                o << "          if (" << (FP && !boxed ? "!(f & 2)" : "!(" + hin + ")")
                  << ") v = sf_ldg_pred(gpl + h" << c << "_g[i], zal && (f & 8));\n";
            } else {
                o << "          T v;\n";
                o << "          if (" << hin << ") v = " << term_expr(halo_operand) << ";\n";
                o << "          else v = sf_ldg_pred(gpl + h" << c << "_g[i], zal && (f & 8));\n";
            }
            if (G.keep == Keep::Smem) {
                Lay self{true, m};
                o << "          " << bname(self, G.lead) << "[h" << c << "_" << lname(self)
                  << "[i]] = v;\n";
            } else {
                o << "          rh" << m << "[i][" << G.depth - 1 << "] = v;\n";
            }
            o << "        }\n";
        }
        if (ready_of[m] >= 0) {
            // this plane of the stage is complete in this CTA: tell the cluster neighbours,
            // wait for theirs, then copy the x-halo columns inside their tiles (same ring
            // layout everywhere: the element TX to the left / right in the neighbour)
            const int r = ready_of[m];
            Lay self{true, m};
            const std::string S = bname(self, G.lead);
            o << "        {  // DSMEM x-halo exchange of this stage's plane\n";
            o << "          if (crank > 0) sf_mbar_arrive_remote(sf_mapa(&cready[" << r << "], crank - 1));\n";
            o << "          if (crank < CX - 1) sf_mbar_arrive_remote(sf_mapa(&cready[" << r << "], crank + 1));\n";
            o << "          sf_mbar_wait_cluster(&cready[" << r << "], cph" << r << ");\n";
            o << "          cph" << r << " ^= 1u;\n";
            if (nh[c]) {
                o << "          #pragma unroll\n          for (int i = 0; i < " << hp[c] << "; ++i) {\n";
                o << "            const int f = h" << c << "_f[i], e = h" << c << "_" << lname(self) << "[i];\n";
                o << "            if (f & 16) " << S << "[e] = sf_ld_dsmem(sf_mapa(" << S << " + e + TX, crank - 1), T(0));\n";
                o << "            else if (f & 32) " << S << "[e] = sf_ld_dsmem(sf_mapa(" << S << " + e - TX, crank + 1), T(0));\n";
                o << "          }\n";
            }
            o << "        }\n";
        }
        o << "      }\n    }\n";
        if (G.keep == Keep::Smem) dirty.insert(m);
    }
    };
    if (spec) {
        o << "    if (tile_in && k >= sf_k0 && k < sf_k1) {\n";
        emit_body(true);
        o << "    } else {\n";
        emit_body(false);
        o << "    }\n";
    } else {
        emit_body(false);
    }
    if (tma) {
        if (L.pbar) {
            o << "    sf_bar_arrive(2 + ((k - KF) & " << NE - 1 << "), NT + 32);  // slots of step k are free\n";
        } else {
            o << "    __syncwarp();\n";
            o << "    if ((tid & 31) == 0) sf_mbar_arrive(&empty[(k - KF) & " << NE - 1 << "]);\n";
        }
    } else {
        o << "    sf_bar_sync(1, NT);\n";
    }
    o << "  }\n";
    if (L.xp) {
        // completion: the last CTA publishes seq to itself and to both neighbours
        // only the end chunks push or read pushed planes: they alone fence at system
        // scope before their CTA's completion (a middle chunk's stores are ordered for
        // this rank's next launch by stream order)
        o << "  if (xs_bot || xs_top) {\n";
        o << "    __threadfence_system();  // this thread's stores (incl. peer pushes) first\n";
        o << "    sf_bar_sync(1, NT);  // the compute threads' barrier (ptxas: no extra barrier)\n  }\n";
        if (std::getenv("SF_DEBUG_XP"))
            o << "  if (tid == 0) printf(\"[" << L.fn << "] own=%p seq=%llu Z0=%d done\\n\", p.xs_own, xs_seq, Z0);\n";
        if (L.xp_dw > 0) {
            // the end chunks facing a neighbour publish to it as soon as they are all done
            o << "  if (tid == 0 && (xs_bot || xs_top)) {\n";
            o << "    int nb = 0, nt = 0;  // end chunks of this launch, per side\n";
            o << "    for (int c = 0; c < (int)gridDim.z; ++c) {\n";
            o << "      const int l = c < p.n_lo, z0 = l ? p.z_base + c * ZC : p.z_hi + (c - p.n_lo) * ZC;\n";
            o << "      const int n = min(ZC, (l ? p.z_mid : p.z_end) - z0);\n";
            o << "      nb += z0 < " << L.xp_dw << "; nt += z0 + n > NZ - " << L.xp_dw << ";\n";
            o << "    }\n";
            o << "    const unsigned per = gridDim.x * gridDim.y;\n";
            o << "    if (xs_bot && p.xs_dn) sf_xs_signal_side((unsigned *)(p.xs_own + 3) + 1, per * nb, p.xs_dn + 1, xs_seq);\n";
            o << "    if (xs_top && p.xs_up) sf_xs_signal_side((unsigned *)(p.xs_own + 4), per * nt, p.xs_up + 0, xs_seq);\n";
            o << "  }\n";
        }
        o << "  if (tid == 0) sf_xs_signal(p.xs_ctr, gridDim.x * gridDim.y * gridDim.z, p.xs_self, "
             "p.xs_dn, p.xs_up, xs_seq);\n";
    }
    if (CX > 1) o << "  sf_cluster_sync();\n";
    o << "}\n";
    L.source = o.str();
    std::ostringstream tbl;
    tbl << "__constant__ T SFK[" << std::max<size_t>(coefs.size(), 1) << "] = {";
    for (size_t i = 0; i < coefs.size(); ++i) tbl << (i ? ", " : "") << lit(coefs[i], f32);
    if (coefs.empty()) tbl << "0";
    tbl << "};";
    if (cc2) tbl << "\n__constant__ int SFZ[2];  // zero-initialised module global";
    const std::string marker = "/*SF_COEF_TABLE*/";
    L.source.replace(L.source.find(marker), marker.size(), tbl.str());
    return L.source;
}

}  // namespace sf
