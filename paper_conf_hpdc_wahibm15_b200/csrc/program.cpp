// program.cpp — program model, validation, DDG/OEG edges and kernel fission.
//
//  * stencil_program_create copies the operations metadata of every kernel
//    (stencil taps, coefficients, read/write sets — the paper's "operations
//    metadata", §3.2.1, §5.1) and validates it.
//  * Dependency edges (DDG/OEG, §3.2.3, Algorithm 1 read as R9,
//    cycles resolved by host order as R10): every pair of statements s < t in
//    program order touching a common array with at least one write.
//  * Fission (§4.1, Algorithm 2, reading R8): connected components
//    of the graph joining each statement's output with the arrays it reads.
#include <algorithm>
#include <cstring>
#include <numeric>

#include "sf_internal.h"

namespace sf {

static int64_t round_up(int64_t v, int64_t m) { return (v + m - 1) / m * m; }

void build_edges(stencil_program *p) {
    p->edges.clear();
    const int n = (int)p->stmts.size();
    // read/write sets per statement
    std::vector<std::vector<int>> reads(n);
    for (int s = 0; s < n; ++s) {
        for (const Term &t : p->stmts[s].terms) {
            reads[s].push_back(t.a.arr);
            if (t.has_b) reads[s].push_back(t.b.arr);
        }
        std::sort(reads[s].begin(), reads[s].end());
        reads[s].erase(std::unique(reads[s].begin(), reads[s].end()), reads[s].end());
    }
    auto has = [](const std::vector<int> &v, int a) {
        return std::binary_search(v.begin(), v.end(), a);
    };
    for (int s = 0; s < n; ++s) {
        const int ws = p->stmts[s].out;
        for (int t = s + 1; t < n; ++t) {
            const int wt = p->stmts[t].out;
            int kind = 0, arr = 1 << 30;
            if (has(reads[t], ws)) { kind |= 1; arr = std::min(arr, ws); }       // RAW
            if (has(reads[s], wt)) { kind |= 2; arr = std::min(arr, wt); }       // WAR
            if (ws == wt) { kind |= 4; arr = std::min(arr, ws); }                // WAW
            if (kind) p->edges.push_back(sp_edge{s, t, kind, arr});
        }
    }
}

std::vector<int> fission_components(const stencil_program *p, int kernel, int *n_comp) {
    const Kernel &K = p->kernels[kernel];
    const int na = (int)p->arrays.size();
    std::vector<int> parent(na);
    std::iota(parent.begin(), parent.end(), 0);
    auto find = [&](int a) {
        while (parent[a] != a) a = parent[a] = parent[parent[a]];
        return a;
    };
    auto unite = [&](int a, int b) { parent[find(a)] = find(b); };
    // dependencyExists(D_i, D_j) (Alg. 2 line 7): an instruction touching one
    // affects the other — here: out <- every array the statement reads.
    for (int gid : K.stmts) {
        const Stmt &S = p->stmts[gid];
        for (const Term &t : S.terms) {
            unite(S.out, t.a.arr);
            if (t.has_b) unite(S.out, t.b.arr);
        }
    }
    // enumerate disconnected subgraphs (Alg. 2 lines 12-19); pieces ordered
    // by their first statement (the random root only permutes them).
    std::map<int, int> comp_id;
    std::vector<int> comp(K.stmts.size());
    for (size_t i = 0; i < K.stmts.size(); ++i) {
        int r = find(p->stmts[K.stmts[i]].out);
        auto it = comp_id.find(r);
        if (it == comp_id.end()) it = comp_id.emplace(r, (int)comp_id.size()).first;
        comp[i] = it->second;
    }
    *n_comp = (int)comp_id.size();
    return comp;
}

}  // namespace sf

using namespace sf;

static void check_tap(const stencil_program *p, const sp_tap &t, const char *where) {
    const int na = (int)p->arrays.size();
    if (t.array < 0 || t.array >= na)
        fail(SP_E_PROGRAM, std::string(where) + ": tap array index out of range");
    const int *g = p->grid.ghost;
    if (std::abs(t.dx) > g[0] || std::abs(t.dy) > g[1] || std::abs(t.dz) > g[2])
        fail(SP_E_PROGRAM, std::string(where) + ": tap offset (" + std::to_string(t.dx) + "," +
                               std::to_string(t.dy) + "," + std::to_string(t.dz) +
                               ") exceeds the ghost width");
}

stencil_program *sf_program_create_impl(const sp_grid *grid, int32_t n_arrays,
                                        const sp_array_desc *arrays, int32_t n_kernels,
                                        const sp_kernel *kernels, sp_comm *comm) {
    if (!grid || n_arrays <= 0 || !arrays || n_kernels <= 0 || !kernels)
        fail(SP_E_ARG, "stencil_program_create: null or empty description");
    std::unique_ptr<stencil_program> p(new stencil_program());
    p->grid = *grid;
    sp_grid &g = p->grid;
    if (g.dtype != SP_F32 && g.dtype != SP_F64) fail(SP_E_ARG, "dtype must be SP_F32 or SP_F64");
    p->elem = (int)g.dtype;
    if (g.nx <= 0 || g.ny <= 0 || g.nz_local <= 0) fail(SP_E_ARG, "grid sizes must be positive");
    if (g.nz_global <= 0) g.nz_global = g.nz_local;
    if (g.nz_global < g.nz_local || g.z_offset < 0 || g.z_offset + g.nz_local > g.nz_global)
        fail(SP_E_ARG, "inconsistent nz_global / z_offset");
    for (int d = 0; d < 3; ++d)
        if (g.ghost[d] < 0 || g.ghost[d] > 16) fail(SP_E_ARG, "ghost width must be in [0,16]");
    if (g.zhalo == 0) g.zhalo = g.ghost[2];
    if (g.zhalo < g.ghost[2] || g.zhalo > 64) fail(SP_E_ARG, "zhalo must be in [ghost_z, 64]");
    if (g.nx > (1 << 24) || g.ny > (1 << 24) || g.nz_local > (1 << 24))
        fail(SP_E_ARG, "grid dimension too large");
    if (comm && (comm->nranks > 1) && g.nz_local < g.zhalo)
        fail(SP_E_ARG, "nz_local must be >= zhalo on several ranks");
    p->comm = comm;

    for (int a = 0; a < n_arrays; ++a) {
        const sp_array_desc &d = arrays[a];
        if (d.role != SP_IN && d.role != SP_OUT && d.role != SP_INOUT && d.role != SP_TEMP)
            fail(SP_E_ARG, "bad array role");
        p->arrays.push_back(ArrayDesc{d.name ? d.name : ("a" + std::to_string(a)), d.role});
    }
    int gid = 0;
    for (int k = 0; k < n_kernels; ++k) {
        const sp_kernel &K = kernels[k];
        if (K.n_stmts <= 0 || !K.stmts) fail(SP_E_PROGRAM, "kernel without statements");
        Kernel kk;
        kk.name = K.name ? K.name : ("K" + std::to_string(k));
        // loop bounds (R2'): default the whole global interior
        int64_t box[6] = {0, g.nx, 0, g.ny, 0, g.nz_global};
        bool boxed = false;
        if (K.box) {
            for (int d = 0; d < 6; ++d) box[d] = K.box[d];
            for (int d = 0; d < 3; ++d) {
                const int64_t hi = d == 0 ? g.nx : d == 1 ? g.ny : g.nz_global;
                if (box[2 * d] < 0 || box[2 * d] > box[2 * d + 1] || box[2 * d + 1] > hi)
                    fail(SP_E_PROGRAM, kk.name + ": box outside the interior or inverted");
            }
            boxed = box[0] != 0 || box[1] != g.nx || box[2] != 0 || box[3] != g.ny ||
                    box[4] != 0 || box[5] != g.nz_global;
        }
        std::vector<int> written;
        for (int s = 0; s < K.n_stmts; ++s) {
            const sp_stmt &S = K.stmts[s];
            if (S.out < 0 || S.out >= n_arrays) fail(SP_E_PROGRAM, kk.name + ": bad output array");
            if (p->arrays[S.out].role == SP_IN)
                fail(SP_E_PROGRAM, kk.name + ": writes array '" + p->arrays[S.out].name +
                                       "' whose role is IN");
            if (S.n_terms <= 0 || !S.terms) fail(SP_E_PROGRAM, kk.name + ": statement without terms");
            Stmt st;
            st.kernel = k;
            st.local = s;
            st.gid = gid++;
            st.out = S.out;
            std::copy(box, box + 6, st.box);
            st.boxed = boxed;
            for (int t = 0; t < S.n_terms; ++t) {
                const sp_term &T = S.terms[t];
                check_tap(p.get(), T.a, kk.name.c_str());
                if (T.has_b) check_tap(p.get(), T.b, kk.name.c_str());
                Term tm;
                // coefficients are rounded to the program dtype once (R4)
                tm.coef = (g.dtype == SP_F32) ? (double)(float)T.coef : T.coef;
                tm.a = Tap{T.a.array, T.a.dx, T.a.dy, T.a.dz};
                tm.has_b = T.has_b != 0;
                tm.b = tm.has_b ? Tap{T.b.array, T.b.dx, T.b.dy, T.b.dz} : Tap{0, 0, 0, 0};
                st.terms.push_back(tm);
            }
            written.push_back(S.out);
            kk.stmts.push_back(st.gid);
            p->stmts.push_back(std::move(st));
        }
        // R3: inside a kernel, an array the kernel writes may only be read at offset 0
        for (int sg : kk.stmts) {
            for (const Term &t : p->stmts[sg].terms) {
                for (int w = 0; w < 2; ++w) {
                    if (w == 1 && !t.has_b) continue;
                    const Tap &tp = w ? t.b : t.a;
                    bool wr = std::find(written.begin(), written.end(), tp.arr) != written.end();
                    if (wr && (tp.dx || tp.dy || tp.dz))
                        fail(SP_E_PROGRAM, kk.name + ": reads '" + p->arrays[tp.arr].name +
                                               "', which it also writes, at a non-zero offset "
                                               "(in-kernel race, reading R3)");
                }
            }
        }
        p->kernels.push_back(std::move(kk));
    }

    // layout: x rows padded to 128 B, interior start aligned to 128 B
    const int64_t per128 = 128 / p->elem;
    sp_layout &L = p->layout;
    L.origin_x = round_up(std::max(g.ghost[0], 1), per128);
    if (g.ghost[0] == 0) L.origin_x = 0;
    L.x_pitch = round_up(L.origin_x + g.nx + g.ghost[0], per128);
    L.origin_y = g.ghost[1];
    L.y_alloc = g.ny + 2 * g.ghost[1];
    L.origin_z = g.zhalo;
    L.z_alloc = g.nz_local + 2 * g.zhalo;
    L.bytes = L.x_pitch * L.y_alloc * L.z_alloc * p->elem;
    p->plane = L.x_pitch * L.y_alloc;
    p->zint_lo = -g.z_offset;
    p->zint_hi = g.nz_global - g.z_offset;
    p->ptrs.assign(n_arrays, nullptr);
    p->peer.assign(n_arrays, {nullptr, nullptr});
    build_edges(p.get());
    return p.release();
}
