// search.cpp — lazy-fission plan search.
//
// The paper's search step (§3.2.4; §4.1): a grouping genetic
// algorithm over kernel fusions whose objective is a performance projection built
// on empirically measured metadata (§3.2.1), with
//   * lazy fission: the fissioned pieces' metadata is gathered in a pre-step, the
//     search starts from the ORIGINAL kernels, and fission is applied when a
//     candidate sits on the shared-memory capacity boundary;
//   * the dynamic penalty f_p(x) = f(x) + sum_i C_i delta_i - C_SM delta_SM
//     (P:L199-211), where C_SM > 0 if fission can relax a violated shared-memory
//     constraint and C_SM < 0 if it cannot.
// The objective is a black box returning a group's time: this library's
// launch-time model (host only) or the group measured on the device (JIT + CUDA
// events), memoised per (members, live-out set).  An exact DP over contiguous
// segmentations of the original kernels seeds the GA: the live-out set (R6) of a
// contiguous group depends on the group alone, so that DP is exact for its space.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstring>
#include <map>
#include <set>

#include "sf_internal.h"

namespace sf {

namespace {

using Key = std::pair<std::vector<int>, std::vector<int>>;  // (member gids, stored gids)
struct Eval {
    double t = 0;  // seconds
    int viol = 0;  // 0 ok, 1 in-group hazard (R11 / R2'), 2 resources (shared memory, registers)
};

class Objective {
  public:
    explicit Objective(stencil_program *p) : p_(p) {}
    virtual ~Objective() = default;
    void prepare(const std::vector<Key> &keys) {
        std::vector<Key> todo;
        std::set<Key> seen;
        for (const Key &k : keys)
            if (!cache_.count(k) && seen.insert(k).second) todo.push_back(k);
        if (!todo.empty()) evaluate(todo);
    }
    const Eval &get(const Key &k) {
        auto it = cache_.find(k);
        if (it == cache_.end()) {
            prepare({k});
            it = cache_.find(k);
        }
        return it->second;
    }
    int evaluated() const { return (int)cache_.size(); }
    // configuration the objective's time was obtained with (zeros: the chooser's)
    sp_tile_config config(const Key &k) const {
        auto it = cfg_.find(k);
        if (it != cfg_.end()) return it->second;
        sp_tile_config c;
        std::memset(&c, 0, sizeof c);
        return c;
    }

  protected:
    virtual void evaluate(const std::vector<Key> &todo) = 0;
    // group analysis + tile choice (pinned to `pin` when given, as sp_plan_tune does);
    // false (with e.viol set) if the group is illegal or the pin does not fit
    bool configure(const Key &k, Launch &L, Eval &e, bool quick, const sp_tile_config *pin = nullptr) {
        const std::set<int> st(k.second.begin(), k.second.end());
        const Options saved = p_->opt;
        try {
            L = analyze_group(p_, k.first, st);
            if (L.dead) return false;
            if (pin) {
                if (pin->tile_x) p_->opt.tile_x = pin->tile_x;
                if (pin->tile_y) p_->opt.tile_y = pin->tile_y;
                if (pin->zchunk) p_->opt.zchunk = pin->zchunk;
                if (pin->threads) p_->opt.threads = pin->threads;
                if (pin->prefetch) p_->opt.prefetch = pin->prefetch;
                if (pin->block_x) p_->opt.block_x = pin->block_x;
                if (pin->block_y) p_->opt.block_y = pin->block_y;
                if (pin->block_cby) p_->opt.block_cby = pin->block_cby;
                if (pin->zqueue) p_->opt.zqueue = pin->zqueue - 1;
                if (pin->fastpath) L.fastpath = pin->fastpath - 1;
                if (pin->frame) L.frame_pin = pin->frame - 1;
            }
            choose_config(p_, L, quick);
            p_->opt = saved;
            model(p_, L);
            return true;
        } catch (const Error &er) {
            p_->opt = saved;
            e.viol = er.code == SP_E_PLAN_HAZARD ? 1 : 2;
            return false;
        }
    }
    stencil_program *p_;
    std::map<Key, Eval> cache_;
    std::map<Key, sp_tile_config> cfg_;
};

// the library's launch-time model (plan.cpp::choose_config), + 3 us per launch
class ModelObjective : public Objective {
  public:
    using Objective::Objective;

  protected:
    void evaluate(const std::vector<Key> &todo) override {
        for (const Key &k : todo) {
            Eval e;
            Launch L;
            if (configure(k, L, e, true)) e.t = L.t_model + 3e-6;
            cache_[k] = e;
        }
    }
};

// measured on the device: every new group of a batch is generated at the chooser's
// configuration and at each candidate configuration that fits, JIT-compiled (in
// parallel), loaded and timed with CUDA events on the caller's stream — median of
// `reps` launches, each after a 256 MB memset that evicts the L2; a group's time is
// its fastest configuration (the paper's per-kernel block tuning, §4.2, folded
// into the objective), remembered for the returned plan
class MeasuredObjective : public Objective {
  public:
    MeasuredObjective(stencil_program *p, void *stream, int reps, std::vector<sp_tile_config> cands)
        : Objective(p), stream_((cudaStream_t)stream), reps_(std::max(1, reps)), cands_(std::move(cands)) {}
    ~MeasuredObjective() override {
        if (flush_) cudaFree(flush_);
        if (ev_[0]) cudaEventDestroy(ev_[0]);
        if (ev_[1]) cudaEventDestroy(ev_[1]);
    }

  protected:
    void evaluate(const std::vector<Key> &todo) override {
        ensure_cuda();
        Mode m;
        std::vector<std::pair<size_t, sp_tile_config>> owner;  // (key index, configuration)
        for (size_t i = 0; i < todo.size(); ++i) {
            Eval e;
            bool any = false;
            for (int v = -1; v < (int)cands_.size(); ++v) {
                Launch L;
                Eval ev;
                if (!configure(todo[i], L, ev, false, v < 0 ? nullptr : &cands_[v])) {
                    if (v < 0) e = ev;  // the chooser's verdict (hazard / no tile fits)
                    if (v < 0 && (ev.viol || L.dead)) break;
                    continue;
                }
                sp_tile_config c;
                std::memset(&c, 0, sizeof c);
                c.tile_x = L.tx; c.tile_y = L.ty; c.zchunk = L.zc; c.threads = L.nt; c.prefetch = L.pf;
                c.block_x = L.vx; c.block_y = L.vy; c.block_cby = L.cby;
                c.fastpath = L.fastpath >= 0 ? L.fastpath + 1 : 0;
                c.frame = L.fr ? 2 : 1;
                bool dup = false;
                for (const auto &o : owner)
                    dup |= o.first == i && !std::memcmp(&o.second, &c, sizeof c);
                if (dup) continue;
                L.name = "search" + std::to_string(i);
                generate_launch(p_, L, (int)m.launches.size(), true);
                m.launches.push_back(std::move(L));
                owner.push_back({i, c});
                any = true;
            }
            if (!any) cache_[todo[i]] = e;
        }
        if (m.launches.empty()) return;
        m.analyzed = true;
        struct Unload {  // modules of this batch are unloaded on every exit path
            Mode &m;
            ~Unload() { unload_mode(m); }
        } unload{m};
        compile_mode(p_, m);
        load_mode(p_, m);
        if (!flush_) {
            if (cudaMalloc(&flush_, kFlush) != cudaSuccess) fail(SP_E_CUDA, "search: flush buffer");
            if (cudaEventCreate(&ev_[0]) != cudaSuccess || cudaEventCreate(&ev_[1]) != cudaSuccess)
                fail(SP_E_CUDA, "search: events");
        }
        for (size_t j = 0; j < m.launches.size(); ++j) {
            launch(p_, m, (int)j, stream_);  // first use (module, descriptors)
            std::vector<float> ts;
            auto ck = [&](cudaError_t e, const char *what) {
                if (e != cudaSuccess)
                    fail(SP_E_CUDA, std::string("search: ") + what + " (" + m.launches[j].fn + ", tile " +
                                        std::to_string(m.launches[j].tx) + "x" + std::to_string(m.launches[j].ty) +
                                        "): " + cudaGetErrorString(e));
            };
            for (int r = 0; r < reps_; ++r) {
                float ms = 0;
                ck(cudaMemsetAsync(flush_, r & 0xff, kFlush, stream_), "L2 flush");
                ck(cudaEventRecord(ev_[0], stream_), "event record");
                launch(p_, m, (int)j, stream_);
                ck(cudaEventRecord(ev_[1], stream_), "event record");
                ck(cudaEventSynchronize(ev_[1]), "kernel");
                ck(cudaEventElapsedTime(&ms, ev_[0], ev_[1]), "elapsed");
                ts.push_back(ms);
            }
            std::sort(ts.begin(), ts.end());
            const double t = ts[ts.size() / 2] * 1e-3;
            const Key &k = todo[owner[j].first];
            auto it = cache_.find(k);
            if (it == cache_.end() || t < it->second.t) {
                Eval e;
                e.t = t;
                cache_[k] = e;
                cfg_[k] = owner[j].second;
            }
        }
    }

  private:
    static constexpr size_t kFlush = 256u << 20;
    cudaStream_t stream_;
    int reps_;
    std::vector<sp_tile_config> cands_;
    void *flush_ = nullptr;
    cudaEvent_t ev_[2] = {nullptr, nullptr};
};

uint64_t splitmix(uint64_t &s) {
    s += 0x9E3779B97F4A7C15ull;
    uint64_t z = s;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

}  // namespace

std::vector<std::vector<int>> search_plan(stencil_program *p, const sp_search_options &opt, void *stream,
                                          sp_search_report *rep, std::vector<sp_tile_config> *configs) {
    std::unique_ptr<Objective> obj;
    if (opt.objective == 1)
        obj.reset(new MeasuredObjective(p, stream, opt.reps > 0 ? opt.reps : 5,
                                        std::vector<sp_tile_config>(opt.configs, opt.configs + std::max(0, opt.n_configs))));
    else obj.reset(new ModelObjective(p));
    const int K = (int)p->kernels.size();
    const int U = opt.max_group_kernels > 0 ? opt.max_group_kernels : 8;
    const double Cv = opt.c_violation > 0 ? opt.c_violation : 1.0;
    const double Csm = opt.c_sm > 0 ? opt.c_sm : 0.5;

    // units = fission pieces (Algorithm 2) in program order
    const std::vector<std::vector<int>> units = fission_units(p);
    const int nu = (int)units.size();
    std::vector<int> unit_kernel(nu), unit_of(p->stmts.size(), -1);
    std::vector<std::vector<int>> kunits(K);
    for (int u = 0; u < nu; ++u) {
        unit_kernel[u] = p->stmts[units[u][0]].kernel;
        kunits[unit_kernel[u]].push_back(u);
        for (int gid : units[u]) unit_of[gid] = u;
    }
    auto sorted = [](std::vector<int> v) {
        std::sort(v.begin(), v.end());
        return v;
    };
    // keys of a plan (groups in execution order) under its live-out sets (R6)
    auto plan_keys = [&](const std::vector<std::vector<int>> &gs) {
        std::vector<std::set<int>> stored;
        live_out(p, true, gs, stored);
        std::vector<Key> keys;
        for (size_t g = 0; g < gs.size(); ++g)
            keys.push_back({sorted(gs[g]), std::vector<int>(stored[g].begin(), stored[g].end())});
        return keys;
    };
    // a contiguous group's key (its live-out set depends on the group alone)
    auto segment_key = [&](const std::vector<int> &mem) {
        std::vector<int> before, after;
        std::set<int> in(mem.begin(), mem.end());
        for (int s = 0; s < (int)p->stmts.size(); ++s)
            if (!in.count(s)) (s < mem.front() ? before : after).push_back(s);
        std::vector<std::vector<int>> gs;
        if (!before.empty()) gs.push_back(before);
        gs.push_back(mem);
        if (!after.empty()) gs.push_back(after);
        return plan_keys(gs)[before.empty() ? 0 : 1];
    };

    // ---- 1. metadata pre-step: every original kernel and every fission piece alone
    std::vector<Key> pre;
    std::vector<Key> kkey(K), ukey(nu);
    for (int k = 0; k < K; ++k) pre.push_back(kkey[k] = segment_key(sorted(p->kernels[k].stmts)));
    for (int u = 0; u < nu; ++u) pre.push_back(ukey[u] = segment_key(sorted(units[u])));
    obj->prepare(pre);
    std::vector<double> tk(K), tu(nu);
    double unfused = 0;
    for (int u = 0; u < nu; ++u) tu[u] = obj->get(ukey[u]).t;
    for (int k = 0; k < K; ++k) {
        const Eval &e = obj->get(kkey[k]);
        double s = 0;
        for (int u : kunits[k]) s += tu[u];
        tk[k] = e.viol ? s : e.t;  // an infeasible kernel is charged its pieces
        unfused += tk[k];
    }
    const double U0 = std::max(unfused, 1e-9);

    // ---- 2. exact DP over contiguous segmentations of the original kernels
    std::vector<std::vector<Key>> seg(K + 1);  // seg[i][l-1]: kernels [i-l, i)
    {
        std::vector<Key> all;
        for (int i = 1; i <= K; ++i)
            for (int l = 1; l <= std::min(U, i); ++l) {
                std::vector<int> mem;
                for (int k = i - l; k < i; ++k) mem.insert(mem.end(), p->kernels[k].stmts.begin(), p->kernels[k].stmts.end());
                seg[i].push_back(segment_key(sorted(mem)));
                all.push_back(seg[i].back());
            }
        obj->prepare(all);
    }
    std::vector<double> best(K + 1, 1e300);
    std::vector<int> from(K + 1, -1);
    best[0] = 0;
    for (int i = 1; i <= K; ++i)
        for (int l = 1; l <= std::min(U, i); ++l) {
            const Eval &e = obj->get(seg[i][l - 1]);
            const double c = e.viol ? (l == 1 ? tk[i - 1] + Cv * U0 : 1e300) : e.t;
            if (best[i - l] + c < best[i]) {
                best[i] = best[i - l] + c;
                from[i] = i - l;
            }
        }
    std::vector<std::vector<int>> dp_plan;
    for (int i = K; i > 0; i = from[i]) {
        std::vector<int> mem;
        for (int k = from[i]; k < i; ++k) mem.insert(mem.end(), p->kernels[k].stmts.begin(), p->kernels[k].stmts.end());
        dp_plan.insert(dp_plan.begin(), sorted(mem));
    }

    // ---- 3. grouping GA with lazy fission and the dynamic penalty f_p
    std::vector<std::vector<int>> succ(nu);
    for (const sp_edge &e : p->edges) {
        const int a = unit_of[e.from], b = unit_of[e.to];
        if (a != b) succ[a].push_back(b);
    }
    for (auto &v : succ) {
        std::sort(v.begin(), v.end());
        v.erase(std::unique(v.begin(), v.end()), v.end());
    }
    uint64_t rs = opt.seed * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull;
    auto rnd = [&](int n) { return (int)(splitmix(rs) % (uint64_t)std::max(n, 1)); };
    struct Chrom {
        std::vector<int> lab;   // group label per unit
        std::vector<char> fis;  // kernel fissioned (its pieces may part)
        bool operator<(const Chrom &o) const { return std::tie(lab, fis) < std::tie(o.lab, o.fis); }
        bool operator==(const Chrom &o) const { return lab == o.lab && fis == o.fis; }
    };
    auto normalize = [&](Chrom &c) {
        for (int k = 0; k < K; ++k)  // an unfissioned kernel's pieces share a group
            if (!c.fis[k])
                for (int u : kunits[k]) c.lab[u] = c.lab[kunits[k][0]];
        std::map<int, int> ren;
        for (int &l : c.lab) {
            auto it = ren.find(l);
            if (it == ren.end()) it = ren.emplace(l, (int)ren.size()).first;
            l = it->second;
        }
    };
    // groups in a topological order of the quotient (ties: first unit); false if cyclic
    auto decode = [&](const Chrom &c, std::vector<std::vector<int>> &gs) {
        const int ng = *std::max_element(c.lab.begin(), c.lab.end()) + 1;
        std::vector<std::vector<int>> mem(ng);
        for (int u = 0; u < nu; ++u) mem[c.lab[u]].push_back(u);
        std::vector<std::set<int>> gsucc(ng);
        std::vector<int> indeg(ng, 0);
        for (int u = 0; u < nu; ++u)
            for (int v : succ[u])
                if (c.lab[u] != c.lab[v] && gsucc[c.lab[u]].insert(c.lab[v]).second) indeg[c.lab[v]]++;
        std::set<std::pair<int, int>> ready;
        for (int g = 0; g < ng; ++g)
            if (!indeg[g] && !mem[g].empty()) ready.insert({mem[g][0], g});
        gs.clear();
        while (!ready.empty()) {
            const int g = ready.begin()->second;
            ready.erase(ready.begin());
            std::vector<int> gids;
            for (int u : mem[g]) gids.insert(gids.end(), units[u].begin(), units[u].end());
            gs.push_back(sorted(gids));
            for (int h : gsucc[g])
                if (--indeg[h] == 0) ready.insert({mem[h][0], h});
        }
        int nonempty = 0;
        for (auto &m : mem) nonempty += !m.empty();
        return (int)gs.size() == nonempty;
    };
    auto keys_of = [&](const Chrom &c, std::vector<Key> &out) {
        std::vector<std::vector<int>> gs;
        if (!decode(c, gs)) return false;
        std::vector<Key> ks = plan_keys(gs);
        out.insert(out.end(), ks.begin(), ks.end());
        return true;
    };
    // f_p: a violating group is charged its units' pre-step times plus C_i; a shared-memory
    // violation is relaxed by C_SM if one of its kernels can still be fissioned, else
    // penalised by it
    auto fitness = [&](const Chrom &c) {
        std::vector<std::vector<int>> gs;
        if (!decode(c, gs)) return unfused + 3 * Cv * U0;  // cyclic group order (OEG violated)
        const std::vector<Key> ks = plan_keys(gs);
        double f = 0, pen = 0;
        for (size_t g = 0; g < gs.size(); ++g) {
            const Eval &e = obj->get(ks[g]);
            if (!e.viol) {
                f += e.t;
                continue;
            }
            bool can_fission = false;
            std::set<int> us;
            for (int gid : gs[g]) us.insert(unit_of[gid]);
            for (int u : us) {
                f += tu[u];
                const int k = unit_kernel[u];
                if (!c.fis[k] && kunits[k].size() > 1) can_fission = true;
            }
            pen += Cv * U0;
            if (e.viol == 2) pen -= (can_fission ? Csm : -Csm) * U0;
        }
        return f + pen;
    };
    auto from_groups = [&](const std::vector<std::vector<int>> &gs) {
        Chrom c;
        c.lab.assign(nu, 0);
        c.fis.assign(K, 0);
        std::vector<int> gof(p->stmts.size());
        for (size_t g = 0; g < gs.size(); ++g)
            for (int gid : gs[g]) gof[gid] = (int)g;
        for (int u = 0; u < nu; ++u) c.lab[u] = gof[units[u][0]];
        for (int k = 0; k < K; ++k)
            for (int u : kunits[k])
                if (c.lab[u] != c.lab[kunits[k][0]]) c.fis[k] = 1;
        normalize(c);
        return c;
    };
    // the movable block of unit u: its whole kernel unless that kernel is fissioned
    auto block = [&](const Chrom &c, int u) {
        const int k = unit_kernel[u];
        return c.fis[k] ? std::vector<int>{u} : kunits[k];
    };
    auto neighbour = [&](const Chrom &c, int u) {  // a unit of the previous / next kernel
        const std::vector<int> b = block(c, u);
        return rnd(2) ? std::max(0, b.front() - 1) : std::min(nu - 1, b.back() + 1);
    };
    auto fission_op = [&](Chrom &c) {
        // lazy fission: a kernel of a group on the shared-memory boundary (viol 2)
        std::vector<std::vector<int>> gs;
        std::vector<int> cand;
        if (decode(c, gs)) {
            const std::vector<Key> ks = plan_keys(gs);
            for (size_t g = 0; g < gs.size(); ++g)
                if (obj->get(ks[g]).viol == 2)
                    for (int gid : gs[g]) {
                        const int k = p->stmts[gid].kernel;
                        if (!c.fis[k] && kunits[k].size() > 1) cand.push_back(k);
                    }
        }
        if (cand.empty()) {  // exploration: fission can also pay by itself
            if (rnd(10)) return;
            for (int k = 0; k < K; ++k)
                if (!c.fis[k] && kunits[k].size() > 1) cand.push_back(k);
            if (cand.empty()) return;
        }
        const int k = cand[rnd((int)cand.size())];
        c.fis[k] = 1;
        const int ng = *std::max_element(c.lab.begin(), c.lab.end()) + 1;
        c.lab[kunits[k].back()] = ng;  // one piece leaves the group
    };
    auto mutate = [&](Chrom &c) {
        const int ng = *std::max_element(c.lab.begin(), c.lab.end()) + 1;
        const int op = rnd(4), u = rnd(nu);
        if (op == 0) {  // merge u's group with a neighbouring block's group
            const int a = c.lab[u], b = c.lab[neighbour(c, u)];
            for (int &l : c.lab)
                if (l == b) l = a;
        } else if (op == 1) {  // split u's group at a cut between blocks
            std::vector<int> mem;
            for (int w = 0; w < nu; ++w)
                if (c.lab[w] == c.lab[u]) mem.push_back(w);
            std::vector<int> cuts;
            for (size_t i = 1; i < mem.size(); ++i)
                if (c.fis[unit_kernel[mem[i]]] || unit_kernel[mem[i]] != unit_kernel[mem[i - 1]])
                    cuts.push_back((int)i);
            if (!cuts.empty()) {
                const int cut = cuts[rnd((int)cuts.size())];
                for (size_t i = cut; i < mem.size(); ++i) c.lab[mem[i]] = ng;
            }
        } else if (op == 2) {  // move u's block to a neighbour's group
            const int to = c.lab[neighbour(c, u)];
            for (int w : block(c, u)) c.lab[w] = to;
        } else {
            fission_op(c);
        }
        normalize(c);
    };
    auto crossover = [&](const Chrom &a, const Chrom &b) {
        Chrom c = a;
        for (int k = 0; k < K; ++k) c.fis[k] = a.fis[k] | b.fis[k];
        int next = *std::max_element(a.lab.begin(), a.lab.end()) + 1;
        const int ngb = *std::max_element(b.lab.begin(), b.lab.end()) + 1;
        for (int g = 0; g < ngb; ++g) {
            if (rnd(2)) continue;
            for (int u = 0; u < nu; ++u)
                if (b.lab[u] == g) c.lab[u] = next;
            ++next;
        }
        normalize(c);
        return c;
    };
    // batch-evaluate the groups of a set of chromosomes (the measured objective compiles
    // them in parallel), then score
    auto score = [&](std::vector<std::pair<double, Chrom>> &pop) {
        std::vector<Key> ks;
        for (auto &x : pop) keys_of(x.second, ks);
        obj->prepare(ks);
        for (auto &x : pop) x.first = fitness(x.second);
    };
    std::vector<std::pair<double, Chrom>> pop;
    const Chrom dp = from_groups(dp_plan);
    pop.push_back({0, dp});
    std::vector<std::vector<int>> perk;
    for (int k = 0; k < K; ++k) perk.push_back(sorted(p->kernels[k].stmts));
    pop.push_back({0, from_groups(perk)});
    pop.push_back({0, from_groups(greedy_plan(p))});
    const int P = std::max(opt.population, 4);
    while ((int)pop.size() < P) {
        Chrom c = dp;
        for (int k = 1 + rnd(4); k > 0; --k) mutate(c);
        pop.push_back({0, c});
    }
    score(pop);
    auto by_fit = [](const std::pair<double, Chrom> &x, const std::pair<double, Chrom> &y) {
        return x.first < y.first || (x.first == y.first && x.second < y.second);
    };
    std::sort(pop.begin(), pop.end(), by_fit);
    auto tournament = [&]() -> const Chrom & {
        int b = rnd((int)pop.size());
        for (int k = 0; k < 2; ++k) b = std::min(b, rnd((int)pop.size()));
        return pop[b].second;
    };
    int gen = 0;
    for (; gen < opt.generations; ++gen) {
        std::vector<std::pair<double, Chrom>> next(pop.begin(), pop.begin() + std::min<size_t>(2, pop.size()));
        std::set<Chrom> seen;
        for (auto &x : next) seen.insert(x.second);
        std::vector<std::pair<double, Chrom>> kids;
        int tries = 0;
        while ((int)(next.size() + kids.size()) < (int)pop.size() && tries++ < 20 * (int)pop.size()) {
            Chrom c = rnd(2) ? crossover(tournament(), tournament()) : tournament();
            for (int k = 1 + rnd(2); k > 0; --k) mutate(c);
            if (!seen.insert(c).second) continue;
            kids.push_back({0, c});
        }
        score(kids);
        next.insert(next.end(), kids.begin(), kids.end());
        std::sort(next.begin(), next.end(), by_fit);
        pop.swap(next);
    }
    std::vector<std::vector<int>> gs;
    decode(pop.front().second, gs);
    if (configs) {
        configs->clear();
        for (const Key &k : plan_keys(gs)) configs->push_back(obj->config(k));
    }
    if (rep) {
        std::memset(rep, 0, sizeof(*rep));
        rep->cost_us = pop.front().first * 1e6;
        rep->dp_cost_us = best[K] * 1e6;
        rep->unfused_cost_us = unfused * 1e6;
        rep->groups_evaluated = obj->evaluated();
        for (int k = 0; k < K; ++k) {
            std::set<int> labs;
            for (int u : kunits[k]) labs.insert(pop.front().second.lab[u]);
            rep->fissioned_kernels += labs.size() > 1;
        }
        rep->generations_run = gen;
    }
    return gs;
}

}  // namespace sf
