// plan.cpp — plan legality, per-launch analysis, tile choice, byte/flop model.
//
// A fused group is the paper's complex fusion (§5.5.3: producers are
// evaluated on extra halo layers before the barrier, consumers on the tile
// after it) combined with simple fusion's input sharing (§5.5.2: each
// array "target of locality" staged on chip once).  On B200 the vertical
// direction is marched ("horizontal mapping to CUDA grid and iterating in the
// vertical direction"): producers run `lead` planes ahead of their
// consumers, so the z-direction needs no recompute inside a chunk.
//
// Readings used: R1 ghost points are loaded, never computed;
// R5 halo depth = accumulated reach per statement; R6 live-out; R7 staging;
// R11 in-group hazards; R12 several writers (SSA inside a group).
#include <algorithm>
#include <climits>
#include <cmath>
#include <cstring>
#include <set>

#include "sf_internal.h"

namespace sf {

static int64_t rup(int64_t v, int64_t m) { return (v + m - 1) / m * m; }

// ----------------------------------------------------------------- analysis
Launch analyze_group(const stencil_program *p, const std::vector<int> &members,
                     const std::set<int> &stored_gids) {
    Launch L;
    L.members = members;
    const int n = (int)members.size();
    L.st.resize(n);
    std::map<int, int> last_writer;   // array -> position
    std::map<int, int> input_of;      // array -> input index
    auto resolve = [&](const Tap &t) {
        auto it = last_writer.find(t.arr);
        if (it != last_writer.end()) return Src{true, it->second, t.dx, t.dy, t.dz};
        auto jt = input_of.find(t.arr);
        if (jt == input_of.end()) {
            jt = input_of.emplace(t.arr, (int)L.in.size()).first;
            Input I;
            I.arr = t.arr;
            L.in.push_back(I);
        }
        return Src{false, jt->second, t.dx, t.dy, t.dz};
    };
    for (int m = 0; m < n; ++m) {
        const Stmt &S = p->stmts[members[m]];
        Stage &G = L.st[m];
        G.gid = S.gid;
        G.out = S.out;
        for (const Term &t : S.terms) {
            TermR r;
            r.coef = t.coef;
            r.a = resolve(t.a);
            r.has_b = t.has_b;
            r.b = t.has_b ? resolve(t.b) : Src{false, -1, 0, 0, 0};
            G.terms.push_back(r);
        }
        last_writer[S.out] = m;
        G.stored = stored_gids.count(S.gid) > 0;
    }

    // backward pass (reading R5): regions, plane ranges, leads
    const int NEG = INT_MIN / 4;
    struct Acc { int ex0, ex1, ey0, ey1, loff, lead, minread; bool any; };
    std::vector<Acc> acc(n, Acc{NEG, NEG, NEG, NEG, INT_MAX / 4, NEG, INT_MAX / 4, false});
    struct IAcc { int ex0, ex1, ey0, ey1, alo, ahi, qlo; bool any; };
    std::vector<IAcc> iacc(L.in.size(), IAcc{NEG, NEG, NEG, NEG, INT_MAX / 4, NEG, INT_MAX / 4, false});
    for (int m = n - 1; m >= 0; --m) {
        Stage &G = L.st[m];
        Acc &A = acc[m];
        if (G.stored) {  // live-out: the tile and the chunk's own planes (R6)
            A.ex0 = std::max(A.ex0, 0); A.ex1 = std::max(A.ex1, 0);
            A.ey0 = std::max(A.ey0, 0); A.ey1 = std::max(A.ey1, 0);
            A.loff = std::min(A.loff, 0); A.lead = std::max(A.lead, 0);
            A.minread = std::min(A.minread, 0);
            A.any = true;
        }
        if (!A.any) continue;  // dead: nothing consumes it
        G.needed = true;
        // every region contains the tile core (the shared thread mapping of the core)
        G.ex0 = std::max(A.ex0, 0); G.ex1 = std::max(A.ex1, 0);
        G.ey0 = std::max(A.ey0, 0); G.ey1 = std::max(A.ey1, 0);
        G.loff = A.loff; G.lead = A.lead;
        G.depth = G.lead - std::min(A.minread, G.lead) + 1;
        for (const TermR &t : G.terms) {
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (s.stage) {
                    Acc &P = acc[s.idx];
                    P.ex0 = std::max(P.ex0, G.ex0 - s.dx); P.ex1 = std::max(P.ex1, G.ex1 + s.dx);
                    P.ey0 = std::max(P.ey0, G.ey0 - s.dy); P.ey1 = std::max(P.ey1, G.ey1 + s.dy);
                    P.loff = std::min(P.loff, G.loff + s.dz);
                    P.lead = std::max(P.lead, G.lead + s.dz);
                    P.minread = std::min(P.minread, G.lead + s.dz);
                    P.any = true;
                } else {
                    IAcc &I = iacc[s.idx];
                    I.ex0 = std::max(I.ex0, G.ex0 - s.dx); I.ex1 = std::max(I.ex1, G.ex1 + s.dx);
                    I.ey0 = std::max(I.ey0, G.ey0 - s.dy); I.ey1 = std::max(I.ey1, G.ey1 + s.dy);
                    I.alo = std::min(I.alo, G.lead + s.dz);
                    I.ahi = std::max(I.ahi, G.lead + s.dz);
                    I.qlo = std::min(I.qlo, G.loff + s.dz);
                    I.any = true;
                }
            }
        }
    }
    // inputs not read by any needed stage are dropped
    std::vector<int> remap(L.in.size(), -1);
    std::vector<Input> ins;
    for (size_t i = 0; i < L.in.size(); ++i) {
        if (!iacc[i].any) continue;
        Input I = L.in[i];
        I.ex0 = iacc[i].ex0; I.ex1 = iacc[i].ex1; I.ey0 = iacc[i].ey0; I.ey1 = iacc[i].ey1;
        I.alo = iacc[i].alo; I.ahi = iacc[i].ahi; I.qlo = iacc[i].qlo;
        remap[i] = (int)ins.size();
        ins.push_back(I);
    }
    for (Stage &G : L.st)
        for (TermR &t : G.terms) {
            if (!t.a.stage) t.a.idx = remap[t.a.idx];
            if (t.has_b && !t.b.stage) t.b.idx = remap[t.b.idx];
        }
    L.in = ins;

    // storage class (reading R7): register if every consumer reads it at
    // (0,0,dz) over exactly its own region, else a shared-memory plane ring
    std::vector<bool> reg_ok(n, true);
    for (int m = 0; m < n; ++m) {
        const Stage &G = L.st[m];
        if (!G.needed) continue;
        for (const TermR &t : G.terms)
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (!s.stage) continue;
                const Stage &P = L.st[s.idx];
                if (s.dx || s.dy || P.ex0 != G.ex0 || P.ex1 != G.ex1 || P.ey0 != G.ey0 ||
                    P.ey1 != G.ey1)
                    reg_ok[s.idx] = false;
            }
    }
    L.kfirst = 0;
    for (int m = 0; m < n; ++m) {
        Stage &G = L.st[m];
        if (!G.needed) { G.keep = Keep::Dead; continue; }
        G.keep = reg_ok[m] ? Keep::Reg : Keep::Smem;
        L.kfirst = std::min(L.kfirst, G.loff - G.lead);
        int c = -1;
        for (size_t i = 0; i < L.cls.size(); ++i)
            if (L.cls[i].x0 == -G.ex0 && L.cls[i].x1 == G.ex1 && L.cls[i].y0 == -G.ey0 &&
                L.cls[i].y1 == G.ey1)
                c = (int)i;
        if (c < 0) {
            c = (int)L.cls.size();
            L.cls.push_back(RegionClass{-G.ex0, G.ex1, -G.ey0, G.ey1});  // x1/y1 are extensions
        }
        G.cls = c;
    }
    L.dead = true;
    for (const Stage &G : L.st) if (G.needed) L.dead = false;

    // z reach for the halo exchange
    L.z_below = 0;
    L.z_above = 0;
    for (const Input &I : L.in) {
        L.z_below = std::max(L.z_below, -I.qlo);
        L.z_above = std::max(L.z_above, I.ahi);
    }

    // R2' (loop bounds): a statement with a sub-box leaves the points outside its
    // box to the array's stored value, which the fused kernel loads from memory;
    // that is the value the original program sees only if no other statement of
    // the group writes the array (before: the stored value would be stale; after:
    // other CTAs would store there while this one loads)
    for (int m = 0; m < n; ++m) {
        const Stage &W = L.st[m];
        if (!p->stmts[W.gid].boxed) continue;
        for (int r = 0; r < n; ++r)
            if (r != m && L.st[r].out == W.out)
                fail(SP_E_PLAN_HAZARD,
                     "statement " + std::to_string(W.gid) + " writes '" + p->arrays[W.out].name +
                         "' over a sub-box of the interior and statement " +
                         std::to_string(L.st[r].gid) + " of the same group also writes it "
                         "(reading R2')");
    }

    // R11: a group must not read from HBM an array it stores, except for a
    // point-wise read of the CTA's own tile and chunk that happens no later
    // than the store.
    for (int m = 0; m < n; ++m) {
        const Stage &W = L.st[m];
        if (!W.stored) continue;
        for (int r = 0; r < n; ++r) {
            const Stage &R = L.st[r];
            if (!R.needed) continue;
            for (const TermR &t : R.terms)
                for (int w = 0; w < 2; ++w) {
                    if (w == 1 && !t.has_b) continue;
                    const Src &s = w ? t.b : t.a;
                    if (s.stage || L.in[s.idx].arr != W.out) continue;
                    // the reader computes exactly the CTA's own tile x chunk (no halo,
                    // no warm-up plane, no plane of the next chunk) and reads the
                    // point it computes; then it reads before any CTA stores there
                    // iff it runs no later than the store: same step (both leads 0)
                    bool ok = s.dx == 0 && s.dy == 0 && s.dz == 0 && R.ex0 == 0 && R.ex1 == 0 &&
                              R.ey0 == 0 && R.ey1 == 0 && R.loff == 0 && R.lead == 0 &&
                              W.lead == 0;
                    // same step: R precedes W in program order, but runs on another
                    // thread when W's region differs from the tile -> barrier first
                    bool ok2 = W.ex0 == 0 && W.ex1 == 0 && W.ey0 == 0 && W.ey1 == 0;
                    if (!ok)
                        fail(SP_E_PLAN_HAZARD,
                             "statement " + std::to_string(R.gid) + " reads '" +
                                 p->arrays[W.out].name + "' from memory while statement " +
                                 std::to_string(W.gid) + " of the same group stores it "
                                 "(reading R11)");
                    if (!ok2) L.st[m].war_barrier = true;
                }
        }
    }
    return L;
}

// -------------------------------------------------------- config and model
struct Cost { double t; int64_t smem; };

static int pow2ceil(int v) {
    int r = 1;
    while (r < v) r <<= 1;
    return r;
}

static void layout_launch(const stencil_program *p, Launch &L) {
    if (L.tx % (16 / p->elem)) fail(SP_E_ARG, "tile_x must be a multiple of 16 bytes");
    const int e = p->elem;
    L.rw_pad = 16 / e;  // TMA: inner box extent multiple of 16 B
    L.in_off.clear(); L.in_plane.clear(); L.in_rw.clear(); L.in_rh.clear(); L.in_depth.clear();
    L.st_off.clear(); L.st_plane.clear(); L.st_w.clear(); L.st_h.clear(); L.st_depth.clear();
    // region-vector evaluation reads up to VW-1+reach elements beyond a layout row's
    // columns at the region edges (lanes whose results are never consumed): guard bands
    // keep those reads inside the allocation
    int64_t off = L.fr ? 256 : 0;
    L.n_bars = 0;
    for (Input &I : L.in) {
        // the innermost start coordinate of a TMA box must be 16-B aligned: the tile
        // origin is, so round the left extension up to 16 B
        I.bx0 = (int)rup(std::max(I.ex0, 0), L.rw_pad);
        int rw = (int)rup(L.tx + I.bx0 + std::max(I.ex1, 0), L.rw_pad);
        int rh = L.ty + I.ey0 + I.ey1;
        // frame mode: a 128-B guard after every plane slot (never written) takes the
        // reads of edge lanes past a row end, so they never touch a slot being refilled
        int64_t plane = rup((int64_t)rw * rh, 128 / e) + (L.fr ? 128 / e : 0);
        int D = I.ahi - I.alo + 1 + L.pf;  // ring slot = plane mod D (constant modulo per step)
        if (p->opt.pow2ring) D = pow2ceil(D);  // slot = a mask instead of a multiply-high modulo
        L.in_off.push_back(off);
        L.in_plane.push_back(plane);
        L.in_rw.push_back(rw);
        L.in_rh.push_back(rh);
        L.in_depth.push_back(D);
        off += plane * D * e;
    }
    L.nbar_full = pow2ceil(L.pf + 1);
    L.nbar_empty = pow2ceil(L.pf + 2);
    L.n_bars = L.nbar_full + L.nbar_empty;
    for (Stage &G : L.st) {
        G.sx0 = (int)rup(G.ex0, L.rw_pad);
        int w = (int)rup(G.sx0 + L.tx + G.ex1, L.rw_pad), h = L.ty + G.ey0 + G.ey1;
        L.st_w.push_back(w);
        L.st_h.push_back(h);
        if (G.keep == Keep::Smem) {
            // one plane deeper than the reuse distance: no end-of-step barrier needed
            int D = G.depth + 1;
            if (p->opt.pow2ring) D = pow2ceil(D);
            int64_t plane = rup((int64_t)w * h, 128 / e) + (L.fr ? 128 / e : 0);
            L.st_off.push_back(off);
            L.st_plane.push_back(plane);
            L.st_depth.push_back(D);
            off += plane * D * e;
        } else {
            L.st_off.push_back(-1);
            L.st_plane.push_back(0);
            L.st_depth.push_back(0);
        }
    }
    if (L.fr) off += 256;
    off = rup(off, 8);
    L.bar_off = off;
    off += 8 * (int64_t)L.n_bars;
    L.ready_off = off;  // cluster plane-ready barriers (option cluster_x), one per smem stage
    for (const Stage &G : L.st) off += G.keep == Keep::Smem ? 8 : 0;
    L.smem = rup(off, 128);
}

// register estimate of a configured launch (occupancy model of the tile chooser;
// the paper tunes block size with the occupancy-calculator equations, §4.2)
static int estimate_regs(const stencil_program *p, const Launch &L) {
    return codegen_regs(p, L);
}

// issued instructions per output point (thread-level), for the issue-rate ceiling
static double estimate_instr(const Launch &L, bool factor) {
    const double tile = (double)L.tx * L.ty;
    double per_pt = codegen_smem_loads(L) * 1.2, per_step = 60;
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        double pts = (double)(L.tx + G.ex0 + G.ex1) * (L.ty + G.ey0 + G.ey1);
        double halo = pts - tile;
        int ops = 0;
        std::vector<const Src *> bs;  // distinct b operands (one multiply each when factored)
        for (const TermR &t : G.terms) {
            ops += 1;
            if (!t.has_b) continue;
            bool seen = false;
            for (const Src *b : bs)
                seen |= b->stage == t.b.stage && b->idx == t.b.idx && b->dx == t.b.dx &&
                        b->dy == t.b.dy && b->dz == t.b.dz;
            if (!factor || !seen) ops += 1;
            bs.push_back(&t.b);
        }
        per_pt += ops + 1 + (G.stored ? 0.5 : 0) + halo / tile * (2 * ops + 10);
        per_step += 12;
    }
    // per-step work is shared by the points of a thread
    return per_pt + per_step * L.nt / tile;
}

// per-point byte/flop model of a configured launch
void model(const stencil_program *p, Launch &L) {
    const int e = p->elem;
    const double tile = (double)L.tx * L.ty * L.zc;
    int n_store = 0;
    double fl_alg = 0, fl_exec = 0, sm = 0;
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        if (G.stored) ++n_store;
        int prods = 0;
        for (const TermR &t : G.terms) prods += t.has_b;
        double f = 2.0 * G.terms.size() - 1 + prods;
        fl_alg += f;
        double pts = (double)(L.tx + G.ex0 + G.ex1) * (L.ty + G.ey0 + G.ey1) *
                     (L.zc - 1 + G.lead - G.loff + 1);
        fl_exec += f * pts / tile;
        int smem_reads = 0;
        for (const TermR &t : G.terms)
            for (int w = 0; w < 2; ++w) {
                if (w == 1 && !t.has_b) continue;
                const Src &s = w ? t.b : t.a;
                if (!s.stage || L.st[s.idx].keep == Keep::Smem) ++smem_reads;
            }
        const double core = (double)L.tx * L.ty * (L.zc - 1 + G.lead - G.loff + 1);
        sm += (smem_reads * (pts - core) + (G.keep == Keep::Smem ? pts : 0)) * e / tile;
    }
    sm += codegen_smem_loads(L) * e;
    double by_exec = n_store * (double)e;
    for (size_t i = 0; i < L.in.size(); ++i) {
        const Input &I = L.in[i];
        double planes = (L.zc - 1 + I.ahi) - I.qlo + 1;
        double b = (double)L.in_rw[i] * L.in_rh[i] * planes * e / tile;
        by_exec += b;
        sm += b;  // TMA writes into shared memory
    }
    L.bytes_alg = (double)e * (L.in.size() + n_store);
    L.flops_alg = fl_alg;
    L.flops_exec = fl_exec;
    L.bytes_exec = by_exec;
    L.smem_pt = sm;
}

static int max_region_points(const Launch &L) {
    int m = 0;
    for (const Stage &G : L.st)
        if (G.needed) m = std::max(m, (L.tx + G.ex0 + G.ex1) * (L.ty + G.ey0 + G.ey1));
    return m;
}

// Region-vector evaluation ("frame"): needs the TMA loader and no per-statement loop
// boxes; peer push and clusters keep the block form (their codegen assumes it).
static bool frame_eligible(const stencil_program *p, const Launch &L) {
    if (p->opt.loader != 0 || p->opt.xpush || p->opt.cluster_x > 1) return false;
    for (const Stage &G : L.st)
        if (G.needed && p->stmts[G.gid].boxed) return false;
    return true;
}

void choose_config(const stencil_program *p, Launch &L, bool quick) {
    const sp_grid &g = p->grid;
    const int e = p->elem;
    const int64_t nz = g.nz_local;
    const Options &o = p->opt;
    const int fmode = L.frame_pin >= 0 ? L.frame_pin : o.frame;
    L.fr = frame_eligible(p, L) && fmode != 0;
    L.fr2 = L.fr && fmode == 2;
    const bool fr = L.fr;
    const int VW = 16 / e;
    std::vector<int> cx, cz, cn, cp, cvx, cvy, ccb, cty;
    if (o.tile_y) cty = {o.tile_y};
    else cty = {4, 8, 16, 32};
    if (o.tile_x) cx = {o.tile_x};
    else if (quick) cx = e == 8 ? std::vector<int>{32, 64} : std::vector<int>{64, 128};
    else cx = e == 8 ? std::vector<int>{16, 32, 64} : std::vector<int>{32, 64, 128};
    if (o.zchunk) cz = {o.zchunk};
    else if (quick) cz = {16, 32};
    else cz = {8, 16, 32};  // measured: longer chunks lose on every C2-C5 group (profiles/sweeps)
    if (o.threads) cn = {o.threads};
    else cn = {64, 128, 256};
    if (o.prefetch >= 0) cp = {o.prefetch};
    else if (quick) cp = {1, 2};
    else cp = {1, 2, 3};
    if (o.block_x) cvx = {o.block_x};
    else cvx = e == 8 ? std::vector<int>{1, 2} : std::vector<int>{1, 2, 4};
    if (o.block_y) cvy = {o.block_y};
    else cvy = {1, 2, 4};
    if (o.block_cby) ccb = {o.block_cby};
    else ccb = {1, 2, 4};
    if (fr) {  // one 16-byte x-vector per evaluation unit; the tile height is free
        cvx = {VW};
        cvy = {1};
        ccb = {1};
    }
    const double sms = p->num_sms;
    const double clk = 1.85e9;
    const double hbm = 6.0e12, smem_bw = sms * 128 * clk;
    const double alu = sms * (e == 8 ? 64 : 128) * clk;
    const double pts = (double)g.nx * g.ny * nz;
    Launch best;
    double best_t = 1e300;
    for (int tx : cx) {
        if (!o.tile_x && tx >= 2 * g.nx && tx != cx.front()) continue;
        for (int vx : cvx) {
            if (tx % vx) continue;
            const int xt = tx / vx;
            for (int nt : cn) {
                if (!fr && (nt % xt || xt > nt)) continue;
                const int yt = fr ? 1 : nt / xt;
                for (int vy : (fr ? cty : cvy))
                    for (int cby : ccb) {
                        const int ty = fr ? vy : yt * vy * cby;
                        if (fr && !o.tile_y && ty >= 2 * g.ny && ty != cty.front()) continue;
                        if (!fr && o.tile_y && ty != o.tile_y) continue;
                        if (!fr && !o.tile_y && (ty > 64 || (ty >= 2 * g.ny && (vy > 1 || cby > 1))))
                            continue;
                        for (int zc : cz) {
                            if (!o.zchunk && zc >= 2 * nz && zc != cz.front()) continue;
                            for (int pf : cp) {
                                Launch C = L;
                                C.tx = tx; C.ty = ty; C.zc = (int)std::min<int64_t>(zc, nz);
                                C.pf = pf; C.nt = nt; C.vx = vx; C.vy = fr ? 1 : vy; C.cby = cby;
                                C.zq = fr ? (L.fr2 ? 2 : 0) : o.zqueue;
                                C.nth = nt + (o.loader == 0 ? 32 : 0);
                                layout_launch(p, C);
                                if (C.smem > 227 * 1024) continue;
                                bool box_ok = true;  // TMA box extents are limited to 256
                                for (size_t i = 0; i < C.in.size(); ++i)
                                    if (C.in_rw[i] > 256 || C.in_rh[i] > 256) box_ok = false;
                                if (!box_ok) continue;
                                C.est_regs = estimate_regs(p, C);
                                const bool forced = o.tile_x && o.block_x && o.block_y && o.block_cby &&
                                                    o.threads;
                                if (C.est_regs > 255 && !forced) continue;
                                model(p, C);
                                const int regs_alloc = (int)rup(std::min(C.est_regs, 255), 8);
                                C.ntx = (int)((g.nx + tx - 1) / tx);
                                C.nty = (int)((g.ny + ty - 1) / ty);
                                C.nch = (int)((nz + C.zc - 1) / C.zc);
                                double ctas = (double)C.ntx * C.nty * C.nch;
                                // registers: per warp in units of 256, each of the 4 SM
                                // sub-partitions holds 16K and a quarter of the warps
                                const int wpc = (C.nth + 31) / 32, rw = regs_alloc * 32 / 256 * 256;
                                int by_regs = 0;
                                for (int c = 1; c <= 32; ++c)
                                    if (((c * wpc + 3) / 4) * rw <= 16384) by_regs = c;
                                int per_sm = (int)std::min<int64_t>(
                                    {(int64_t)(228 * 1024 / (C.smem + 1024)), (int64_t)(2048 / C.nth),
                                     32, (int64_t)by_regs});
                                if (per_sm < 1) continue;
                                // Launch-time model, fitted to measured sweeps of C2/C3/C4/C5
                                // groups (tools/model_fit.py, profiles/sweeps/): the busiest
                                // of HBM, shared memory (80 % of 128 B/clk/SM), FP pipe and
                                // instruction issue, where issue is latency-limited by the
                                // resident compute warps times the ILP of the register block;
                                // HBM is latency-limited below ~1 us of bytes in flight per SM.
                                double slots = sms * per_sm;
                                double waves = std::ceil(ctas / slots);
                                double fill = ctas / (waves * slots);
                                const double res = std::min<double>(per_sm, std::ceil(ctas / sms));
                                double t_mem = C.bytes_exec * pts / hbm;
                                double t_sm = C.smem_pt * pts / (smem_bw * 0.8);
                                double t_alu = C.flops_exec * pts / alu;
                                const double warps = res * nt / 32;
                                const double ilp = fr ? 4.0 : std::min(4, vx * vy * cby);
                                const double ipc = std::min(3.2, warps * std::sqrt(ilp) / 16.0);
                                double t_issue = estimate_instr(C, p->opt.fmad && p->opt.factor) * pts /
                                                 32.0 / (sms * ipc * clk);
                                int n_store = 0;
                                for (const Stage &G : C.st) n_store += G.needed && G.stored;
                                const double inflight = res * (C.bytes_exec - n_store * e) * tx * ty *
                                                        std::max(pf, 1);
                                const double need = hbm / sms * 1e-6;
                                if (inflight < need) t_mem *= need / std::max(inflight, 1.0);
                                double t = std::max({t_mem, t_sm, t_alu, t_issue}) / fill;
                                t += 100e-9 * (C.zc - C.kfirst) * waves;  // per-step march overhead
                                C.t_model = t;
                                if (t < best_t) { best_t = t; best = C; }
                            }
                        }
                    }
            }
        }
    }
    if (best_t >= 1e299 && L.fr2) {
        // frame mode 2's register queues do not fit at any shape: plain frame mode
        Launch R = L;
        R.frame_pin = 1;
        choose_config(p, R, quick);
        L = R;
        return;
    }
    if (best_t >= 1e299)
        fail(SP_E_RESOURCES, "group '" + L.name + "': no tile configuration fits in 227 KB of "
                             "shared memory / 255 registers (split the group: fission/fusion plan)");
    L = best;
}

// ---------------------------------------------------------------- plans
void live_out(const stencil_program *p, bool fused, const std::vector<std::vector<int>> &groups,
              std::vector<std::set<int>> &stored) {
    stored.assign(groups.size(), {});
    const int na = (int)p->arrays.size();
    if (!fused) {
        // original kernel: every array it writes goes to memory (last writer)
        for (size_t g = 0; g < groups.size(); ++g) {
            std::map<int, int> last;
            for (int gid : groups[g]) last[p->stmts[gid].out] = gid;
            for (auto &kv : last) stored[g].insert(kv.second);
        }
        return;
    }
    // reading R6: X written in G is stored iff a later group reads X from
    // memory before any rewrite, or X is OUT/INOUT and G holds its last writer.
    std::vector<std::pair<int, int>> lastw(na, {-1, -1});  // (group, gid)
    for (size_t g = 0; g < groups.size(); ++g) {
        std::set<int> written_here;
        for (int gid : groups[g]) {
            const Stmt &S = p->stmts[gid];
            for (const Term &t : S.terms)
                for (int w = 0; w < 2; ++w) {
                    if (w == 1 && !t.has_b) continue;
                    int a = w ? t.b.arr : t.a.arr;
                    if (written_here.count(a)) continue;  // on-chip value
                    if (lastw[a].first >= 0 && lastw[a].first < (int)g)
                        stored[lastw[a].first].insert(lastw[a].second);
                }
            // R2': a statement with loop bounds overwrites only its box; every other
            // point keeps the previous value, which it loads from memory (codegen) —
            // so a boxed write reads the array like a tap does
            if (S.boxed && !written_here.count(S.out) && lastw[S.out].first >= 0 &&
                lastw[S.out].first < (int)g)
                stored[lastw[S.out].first].insert(lastw[S.out].second);
            written_here.insert(S.out);
        }
        std::map<int, int> last;
        for (int gid : groups[g]) last[p->stmts[gid].out] = gid;
        for (auto &kv : last) lastw[kv.first] = {(int)g, kv.second};
    }
    for (int a = 0; a < na; ++a)
        if ((p->arrays[a].role == SP_OUT || p->arrays[a].role == SP_INOUT) && lastw[a].first >= 0)
            stored[lastw[a].first].insert(lastw[a].second);
}

void analyze_mode(stencil_program *p, bool fused, const std::vector<std::vector<int>> &groups,
                  Mode &out) {
    std::vector<std::set<int>> stored;
    live_out(p, fused, groups, stored);
    Mode m;
    for (size_t g = 0; g < groups.size(); ++g) {
        Launch L = analyze_group(p, groups[g], stored[g]);
        if (fused) {
            L.name = "group" + std::to_string(g);
        } else {
            L.name = p->kernels[p->stmts[groups[g][0]].kernel].name;
        }
        if (p->comm && p->comm->nranks > 1 &&
            (L.z_below > p->grid.zhalo || L.z_above > p->grid.zhalo))
            fail(SP_E_RESOURCES, L.name + ": accumulated z-reach " +
                                     std::to_string(std::max(L.z_below, L.z_above)) +
                                     " exceeds zhalo " + std::to_string(p->grid.zhalo));
        if (!fused) L.frame_pin = 0;  // the "frame" option applies to fused groups (pins to any)
        if (!L.dead) {
            // per-launch tuned configuration (sp_plan_tune) overrides the chooser's search
            auto &tune = fused ? p->tune_fused : p->tune_unfused;
            auto it = tune.find((int)g);
            if (it != tune.end()) {
                Options saved = p->opt;
                const sp_tile_config &c = it->second;
                if (c.tile_x) p->opt.tile_x = c.tile_x;
                if (c.tile_y) p->opt.tile_y = c.tile_y;
                if (c.zchunk) p->opt.zchunk = c.zchunk;
                if (c.threads) p->opt.threads = c.threads;
                if (c.prefetch) p->opt.prefetch = c.prefetch;
                if (c.block_x) p->opt.block_x = c.block_x;
                if (c.block_y) p->opt.block_y = c.block_y;
                if (c.block_cby) p->opt.block_cby = c.block_cby;
                if (c.zqueue) p->opt.zqueue = c.zqueue - 1;
                if (c.fastpath) L.fastpath = c.fastpath - 1;
                if (c.frame) L.frame_pin = c.frame - 1;
                try {
                    choose_config(p, L);
                } catch (...) {
                    p->opt = saved;
                    throw;
                }
                p->opt = saved;
            } else {
                choose_config(p, L);
            }
            model(p, L);
        }
        m.launches.push_back(std::move(L));
    }
    exchange_schedule(p, m);  // also decides the peer pushes codegen emits
    for (size_t i = 0; i < m.launches.size(); ++i)
        if (!m.launches[i].dead) generate_launch(p, m.launches[i], (int)i, fused);
    m.analyzed = true;
    out = std::move(m);
}

void fill_report(const stencil_program *p, const Launch &L, sp_group_report *r) {
    std::memset(r, 0, sizeof(*r));
    for (const Stage &G : L.st) {
        if (!G.needed) continue;
        r->n_stmts++;
        if (G.stored) r->n_stores++;
        if (G.keep == Keep::Smem) r->n_smem_stages++;
        if (G.keep == Keep::Reg) r->n_reg_stages++;
        r->ext[0] = std::max(r->ext[0], G.ex0);
        r->ext[1] = std::max(r->ext[1], G.ex1);
        r->ext[2] = std::max(r->ext[2], G.ey0);
        r->ext[3] = std::max(r->ext[3], G.ey1);
    }
    r->n_inputs = (int)L.in.size();
    r->z_below = L.z_below;
    r->z_above = L.z_above;
    r->tile_x = L.tx;
    r->tile_y = L.ty;
    r->zchunk = L.zc;
    r->threads = L.nt;
    r->grid_ctas = L.ntx * L.nty * L.nch;
    r->regs_per_thread = L.regs;
    r->smem_bytes = L.smem;
    r->bytes_alg = L.bytes_alg;
    r->flops_alg = L.flops_alg;
    r->bytes_exec = L.bytes_exec;
    r->flops_exec = L.flops_exec;
    r->smem_bytes_pt = L.smem_pt;
    r->block_x = L.vx;
    r->block_y = L.vy;
    r->block_cby = L.cby;
    r->t_model_us = L.t_model * 1e6;
    r->zqueue = L.zq;
    r->est_regs = L.est_regs;
    r->warmup_steps = -L.kfirst;
    r->prefetch = L.pf;
    r->instr_pt = L.dead ? 0 : estimate_instr(L, p->opt.fmad && p->opt.factor);
}

}  // namespace sf

// --------------------------------------------------------- plan validation
using namespace sf;

void sf_plan_set_impl(stencil_program *p, int32_t n_groups, const int32_t *group_begin,
                      const sp_stmt_ref *members) {
    if (n_groups <= 0 || !group_begin || !members) fail(SP_E_ARG, "fusion_plan_set: empty plan");
    const int ns = (int)p->stmts.size();
    std::vector<int> group_of(ns, -1);
    std::vector<std::vector<int>> groups(n_groups);
    if (group_begin[0] != 0) fail(SP_E_ARG, "group_begin[0] must be 0");
    for (int g = 0; g < n_groups; ++g) {
        if (group_begin[g + 1] <= group_begin[g]) fail(SP_E_ARG, "empty group in plan");
        for (int i = group_begin[g]; i < group_begin[g + 1]; ++i) {
            const sp_stmt_ref &r = members[i];
            if (r.kernel < 0 || r.kernel >= (int)p->kernels.size())
                fail(SP_E_ARG, "plan member: kernel index out of range");
            const Kernel &K = p->kernels[r.kernel];
            if (r.stmt < 0 || r.stmt >= (int)K.stmts.size())
                fail(SP_E_ARG, "plan member: statement index out of range");
            int gid = K.stmts[r.stmt];
            if (group_of[gid] >= 0)
                fail(SP_E_PLAN_PARTITION, "statement " + K.name + ":" + std::to_string(r.stmt) +
                                              " appears twice in the plan");
            group_of[gid] = g;
            groups[g].push_back(gid);
        }
        std::sort(groups[g].begin(), groups[g].end());  // program order inside a group
    }
    for (int s = 0; s < ns; ++s)
        if (group_of[s] < 0) {
            const Stmt &S = p->stmts[s];
            fail(SP_E_PLAN_PARTITION, "statement " + p->kernels[S.kernel].name + ":" +
                                          std::to_string(S.local) + " is missing from the plan");
        }
    // order: every dependency edge must go forward in the new OEG
    for (const sp_edge &e : p->edges)
        if (group_of[e.from] > group_of[e.to]) {
            const Stmt &A = p->stmts[e.from], &B = p->stmts[e.to];
            fail(SP_E_PLAN_ORDER, "dependency " + p->kernels[A.kernel].name + ":" +
                                      std::to_string(A.local) + " -> " +
                                      p->kernels[B.kernel].name + ":" + std::to_string(B.local) +
                                      " (array '" + p->arrays[e.array].name +
                                      "') runs backwards in the plan");
        }
    Mode m;
    auto saved_tune = p->tune_fused;
    p->tune_fused.clear();  // tuned configurations belong to the previous plan
    try {
        analyze_mode(p, true, groups, m);  // throws on hazards / resources; old plan kept
    } catch (...) {
        p->tune_fused = saved_tune;
        throw;
    }
    unload_mode(p->fused);
    p->fused = std::move(m);
    p->plan_groups = groups;
    p->has_plan = true;
}

// ------------------------------------------------------------ greedy planner
// Host-side plan search (NEXT #1 in SURVEY.md §8(f); the paper's GGA search,
// P:L140 §3.2.4 and P:L274-276 §5.4, evaluates candidate fusions with a
// performance model, penalising infeasible ones).  Units are fission pieces
// (§4.1: a kernel starts fully fissioned); adjacent groups in program
// order are merged greedily while the modelled step time drops.  A candidate
// group that violates a hazard (R11) or fits no tile is infeasible.
namespace sf {
// units of the plan search: fission pieces (§4.1) in program order
std::vector<std::vector<int>> fission_units(const stencil_program *p) {
    std::vector<std::vector<int>> units;
    for (size_t k = 0; k < p->kernels.size(); ++k) {
        int nc = 0;
        std::vector<int> comp = fission_components(p, (int)k, &nc);
        std::vector<std::vector<int>> pieces(nc);
        for (size_t i = 0; i < comp.size(); ++i) pieces[comp[i]].push_back(p->kernels[k].stmts[i]);
        for (auto &pc : pieces) units.push_back(pc);
    }
    return units;
}

// modelled step time of a plan (groups in execution order): sum of the launch-time
// model of every group under its live-out set (reading R6), memoised per group;
// an illegal group (hazard R11, resources) costs 1e30
struct PlanCost {
    stencil_program *p;
    std::map<std::pair<std::vector<int>, std::vector<int>>, double> cache;
    double group(const std::vector<int> &mem, const std::set<int> &stored) {
        std::vector<int> st(stored.begin(), stored.end());
        auto key = std::make_pair(mem, st);
        auto it = cache.find(key);
        if (it != cache.end()) return it->second;
        double c;
        try {
            Launch L = analyze_group(p, mem, stored);
            if (L.dead) c = 0;
            else {
                choose_config(p, L, true);
                c = L.t_model + 3e-6;  // + launch cost
            }
        } catch (const Error &) {
            c = 1e30;
        }
        cache[key] = c;
        return c;
    }
    double plan(const std::vector<std::vector<int>> &gs) {
        std::vector<std::set<int>> stored;
        live_out(p, true, gs, stored);
        double t = 0;
        for (size_t g = 0; g < gs.size() && t < 1e30; ++g) t += group(gs[g], stored[g]);
        return t;
    }
};

std::vector<std::vector<int>> greedy_plan(stencil_program *p) {
    // units: fission pieces in program order
    std::vector<std::vector<int>> groups = fission_units(p);
    PlanCost pc{p, {}};
    auto plan_cost = [&](const std::vector<std::vector<int>> &gs) { return pc.plan(gs); };
    double cur = plan_cost(groups);
    for (;;) {
        double best = cur;
        size_t best_i = 0;
        for (size_t i = 0; i + 1 < groups.size(); ++i) {
            std::vector<std::vector<int>> cand = groups;
            cand[i].insert(cand[i].end(), cand[i + 1].begin(), cand[i + 1].end());
            std::sort(cand[i].begin(), cand[i].end());
            cand.erase(cand.begin() + i + 1);
            double c = plan_cost(cand);
            if (c < best - 1e-9) { best = c; best_i = i; }
        }
        if (best >= cur) break;
        groups[best_i].insert(groups[best_i].end(), groups[best_i + 1].begin(), groups[best_i + 1].end());
        std::sort(groups[best_i].begin(), groups[best_i].end());
        groups.erase(groups.begin() + best_i + 1);
        cur = best;
    }
    return groups;
}

}  // namespace sf

void sf_unfused_prepare(stencil_program *p) {
    if (p->unfused.analyzed) return;
    std::vector<std::vector<int>> groups;
    for (const Kernel &K : p->kernels) groups.push_back(K.stmts);
    analyze_mode(p, false, groups, p->unfused);
}
