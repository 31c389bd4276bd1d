"""Empirical fission/fusion plan search on the GPU (host-side search, NEXT #1).

The paper's search evaluates candidate fusions with a model built on measured
performance data (§3.2.4, §5.1).  Here the objective is measured
directly: every candidate group (contiguous in program order, so its live-out set
does not depend on how the rest is grouped) is timed as a one-group sub-program
whose array roles reproduce its live-out set (R6): arrays it writes that a later
statement reads before any rewrite, or that are OUT/INOUT, become "out"; arrays it
reads from memory become "in"/"inout".  Greedy: start from fission pieces
(§4.1), merge the adjacent pair with the largest measured gain, repeat.

python tools/plan_autotune.py C4 --out configs/c4_plan.json
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402


def statements(prog):
    out = []
    for k in prog["kernels"]:
        for i, s in enumerate(k["stmts"]):
            out.append((f"{k['name']}:{i}", s))
    return out


def reads(s):
    r = []
    for t in s["terms"]:
        r.append(t["a"][0])
        if "b" in t:
            r.append(t["b"][0])
    return r


class Timer:
    def __init__(self, prog, iters=7):
        self.prog = prog
        self.stm = statements(prog)
        self.pos = {ref: i for i, (ref, _) in enumerate(self.stm)}
        self.roles = {a["name"]: a["role"] for a in prog["arrays"]}
        self.cache = {}
        self.iters = iters
        self.dev = torch.device("cuda:0")
        self.flush = torch.ones(32 << 20, dtype=torch.float64, device=self.dev)  # read-only L2 flush
        full = Program(prog)
        full.allocate(self.dev, fill=0.0)
        bench.fill_inputs(full, prog, self.dev, 0, prog["grid"]["ghost"][2])
        self.tensors = full.tensors
        self._full = full

    def subprogram(self, refs):
        idx = sorted(self.pos[r] for r in refs)
        last = idx[-1]
        written, read_mem = set(), set()
        for i in idx:
            s = self.stm[i][1]
            for a in reads(s):
                if a not in written:
                    read_mem.add(a)
            written.add(s["out"])
        later_needed = set()
        seen_write = set()
        for j in range(last + 1, len(self.stm)):
            s = self.stm[j][1]
            for a in reads(s):
                if a in written and a not in seen_write:
                    later_needed.add(a)
            seen_write.add(s["out"])
        used = written | read_mem
        arrays = []
        for a in self.prog["arrays"]:
            n = a["name"]
            if n not in used:
                continue
            out = n in written and (n in later_needed or self.roles[n] in ("out", "inout"))
            if n in written:
                role = ("inout" if n in read_mem else "out") if out else "temp"
            else:
                role = "in"
            arrays.append({"name": n, "role": role})
        kernels = [{"name": f"s{i}", "stmts": [self.stm[i][1]]} for i in idx]
        sub = dict(self.prog, arrays=arrays, kernels=kernels)
        sub["plans"] = {"fused": [[k["name"] for k in kernels]]}
        return sub

    def _timeit(self, p):
        p.run_launch("fused", 0)
        torch.cuda.synchronize()
        ts = []
        for _ in range(self.iters):
            self.flush.sum()
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            p.run_launch("fused", 0)
            e.record()
            torch.cuda.synchronize()
            ts.append(s.elapsed_time(e) * 1e-3)
        return sorted(ts)[len(ts) // 2]

    def time(self, refs):
        """Measured time of a candidate group: the chooser's configuration and the
        hint configurations (winners of earlier tuning), best of them."""
        key = tuple(sorted(refs, key=lambda r: self.pos[r]))
        if key in self.cache:
            return self.cache[key]
        sub = self.subprogram(key)
        t = float("inf")
        try:
            p = Program(sub)
            p.set_plan(sub["plans"]["fused"])
            for a in sub["arrays"]:
                p.bind(a["name"], self.tensors[a["name"]])
            t = self._timeit(p)
            for cfg in self.hints:
                try:
                    p.tune("fused", 0, cfg)
                    t = min(t, self._timeit(p))
                except StencilError:
                    pass
        except StencilError:
            pass
        self.cache[key] = t
        return t

    hints = []


HINTS_F64 = [dict(tile_x=64, tile_y=4, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32),
             dict(tile_x=32, tile_y=8, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32),
             dict(tile_x=32, tile_y=8, threads=256, block_x=1, block_y=1, block_cby=1, zchunk=32)]


def autotune(prog, log=print, max_group=64, hints=True):
    T = Timer(prog)
    if hints and prog["dtype"] == "f64":
        T.hints = HINTS_F64
    full = T._full
    groups = []
    for k in prog["kernels"]:
        comp, n = full.fission(k["name"])
        pieces = [[] for _ in range(n)]
        for i, c in enumerate(comp):
            pieces[c].append(f"{k['name']}:{i}")
        groups += pieces
    cost = [T.time(g) for g in groups]
    log(f"units {len(groups)}  total {sum(cost)*1e3:.3f} ms")
    while True:
        best, bi = 0.0, -1
        for i in range(len(groups) - 1):
            if len(groups[i]) + len(groups[i + 1]) > max_group:
                continue
            t = T.time(groups[i] + groups[i + 1])
            gain = cost[i] + cost[i + 1] - t
            if gain > best:
                best, bi = gain, i
        if bi < 0:
            break
        groups[bi] = groups[bi] + groups[bi + 1]
        cost[bi] = T.time(groups[bi])
        del groups[bi + 1], cost[bi + 1]
        log(f"merge -> {len(groups)} groups, total {sum(cost)*1e3:.3f} ms (gain {best*1e6:.1f} us)")
    return groups, cost


def fission_units(prog, full):
    units = []
    for k in prog["kernels"]:
        comp, n = full.fission(k["name"])
        pieces = [[] for _ in range(n)]
        for i, c in enumerate(comp):
            pieces[c].append(f"{k['name']}:{i}")
        units += pieces
    return units


def dp_segment(prog, log=print, max_units=8, hints=True):
    """Exact optimum over contiguous segmentations of the fission units (the space the
    greedy merges walk) for the same measured objective (sum of isolated group times):
    best[j] = min over i >= j - max_units of best[i] + t(units i..j-1).  Each segment
    is timed once (cached)."""
    T = Timer(prog)
    if hints and prog["dtype"] == "f64":
        T.hints = HINTS_F64
    units = fission_units(prog, T._full)

    def seg(i, j):
        return T.time([r for u in units[i:j] for r in u])

    cuts = segment_dp(len(units), seg, max_units,
                      log=lambda j, b: log(f"prefix {j}/{len(units)}: {b*1e3:.3f} ms "
                                           f"({len(T.cache)} segments timed)"))
    groups = [[r for u in units[i:j] for r in u] for i, j in zip(cuts[:-1], cuts[1:])]
    return groups, [T.time(g) for g in groups]


def segment_dp(n, cost, max_units, log=None):
    """Cut positions 0 = c0 < c1 < ... < ck = n minimising sum cost(c_i, c_i+1) over
    segments of at most max_units units (cost inf: illegal segment)."""
    inf = float("inf")
    best = [0.0] + [inf] * n
    arg = [0] * (n + 1)
    for j in range(1, n + 1):
        for i in range(max(0, j - max_units), j):
            if best[i] == inf:
                continue
            t = cost(i, j)
            if best[i] + t < best[j]:
                best[j], arg[j] = best[i] + t, i
        if log:
            log(j, best[j])
    cuts, j = [n], n
    while j > 0:
        j = arg[j]
        cuts.insert(0, j)
    return cuts


def config_candidates(prog):
    ny = prog["grid"]["ny"]
    tiles = [32, 64] if prog["dtype"] == "f64" else [64, 128]
    out = []
    for tx in tiles:
        for nt in (64, 128, 256):
            for bx, by, cb in ((1, 1, 1), (1, 2, 1), (2, 2, 1), (1, 1, 2), (1, 4, 1), (1, 2, 2),
                               (2, 2, 2), (1, 4, 2), (1, 8, 1)):
                xt = tx // bx
                if nt % xt or xt > nt or bx * by * cb > 8:
                    continue
                ty = nt // xt * by * cb
                if ty > 32 or ty > 2 * ny:
                    continue
                # tall tiles have fewer CTAs: give them shorter z-chunks
                out.append(dict(tile_x=tx, tile_y=ty, threads=nt, block_x=bx, block_y=by,
                                block_cby=cb, zchunk=32 if ty < 16 else 16))
    return out


def tune_configs(prog, groups, tensors, log=print, iters=7):
    """Per-group empirical tile/block tuning (the paper's block-size tuning, §4.2)."""
    dev = torch.device("cuda:0")
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)  # read-only L2 flush (no dirty lines)
    p = Program(prog)
    p.set_plan(groups)
    for n, t in tensors.items():
        p.bind(n, t)

    def timeit(i):
        p.run_launch("fused", i)
        torch.cuda.synchronize()
        ts = []
        for _ in range(iters):
            flush.sum()
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            p.run_launch("fused", i)
            e.record()
            torch.cuda.synchronize()
            ts.append(s.elapsed_time(e) * 1e-3)
        return sorted(ts)[len(ts) // 2]

    best_cfgs = []
    for i in range(len(groups)):
        best, bcfg = timeit(i), None
        cands = config_candidates(prog)
        for cfg in cands:
            try:
                p.tune("fused", i, cfg)
                t = timeit(i)
            except StencilError:
                continue
            if t < best:
                best, bcfg = t, cfg
        if bcfg is not None:
            # refine around the winner: z-chunk, then TMA prefetch distance
            # and step-wide input z-queues (measured slower on C4's flux groups in r1)
            for key, values in (("zchunk", (16, 64)), ("prefetch", (1, 2, 3)), ("zqueue", (2,))):
                base = bcfg
                for v in values:
                    cfg = dict(base, **{key: v})
                    if cfg == base:
                        continue
                    try:
                        p.tune("fused", i, cfg)
                        t = timeit(i)
                    except StencilError:
                        continue
                    if t < best:
                        best, bcfg = t, cfg
        p.tune("fused", i, bcfg)
        best_cfgs.append(bcfg)
        log(f"group {i}: {best*1e6:.1f} us with {bcfg or 'chooser'}")
    return best_cfgs


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--out", default=None)
    ap.add_argument("--tune", action="store_true", help="also tune each group's tile/block config")
    ap.add_argument("--plan-from", default=None, help="skip the search, tune this plan")
    ap.add_argument("--dp", action="store_true", help="exact segmentation DP instead of greedy merges")
    ap.add_argument("--max-units", type=int, default=8, help="DP: fission units per group at most")
    a = ap.parse_args()
    prog = bench.load_workload(a.workload)
    t0 = time.time()
    if a.plan_from:
        groups = json.load(open(a.plan_from))["groups"]
        cost = [0.0] * len(groups)
    elif a.dp:
        groups, cost = dp_segment(prog, log=lambda m: print(m, flush=True), max_units=a.max_units)
    else:
        groups, cost = autotune(prog, log=lambda m: print(m, flush=True))
    print(f"{len(groups)} groups, measured sum {sum(cost)*1e3:.3f} ms, search {time.time()-t0:.0f} s")
    T = Timer(prog, iters=1) if a.tune else None
    cfgs = tune_configs(prog, groups, T.tensors, log=lambda m: print(m, flush=True)) if a.tune else None
    if a.out:
        p = Program(prog)
        p.set_plan(groups)
        fused = sum(r["bytes_alg"] for r in p.reports("fused")) / p.elem
        unfused = sum(r["bytes_alg"] for r in p.reports("unfused")) / p.elem
        planner = "measured segmentation DP" if a.dp else "measured greedy"
        json.dump({"workload": a.workload, "planner": planner + " (tools/plan_autotune.py)",
                   "groups": groups, "group_ms": [c * 1e3 for c in cost], "configs": cfgs,
                   "passes": {"fused": fused, "unfused": unfused}}, open(a.out, "w"), indent=1)
        print("wrote", a.out)


if __name__ == "__main__":
    main()
