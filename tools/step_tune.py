"""In-context tile tuning of a frozen plan (the paper's per-kernel block-size tuning,
P:L251 §4.2), measured the way bench.py measures: whole steps back to back.

python tools/step_tune.py C4 [--out configs/c4_plan.json] [--top 8] [--rounds 1]

Per group: every candidate configuration is timed alone (read-only L2 flush before
each launch) as a prefilter; the best --top of them (plus the current pin) are then
timed inside the step (K steps back to back, the group's neighbours running their
own pinned configurations), and the fastest step wins.  Isolated timing misjudges
groups whose neighbours leave dirty L2 lines or whose tail overlaps the next
group's prologue (PDL), hence the second stage.
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


ZCHUNKS = ()          # () = the default rule (32 planes below 16 rows, else 16)
PREFETCH = (2, 3)


def candidates(ny):
    out = []
    for tx in (32, 64, 128):
        for nt in (64, 128, 256):
            for bx, by, cb in ((1, 1, 1), (1, 2, 1), (2, 2, 1), (1, 1, 2), (1, 4, 1), (1, 2, 2),
                               (2, 2, 2), (1, 4, 2), (1, 8, 1), (2, 4, 1)):
                xt = tx // bx
                if tx % bx or nt % xt or xt > nt or bx * by * cb > 8:
                    continue
                ty = nt // xt * by * cb
                if ty > ny:
                    continue
                # prefetch 1 frees ring planes for more resident CTAs; short chunks add
                # warm-up planes but more CTAs (measured on C2: 32x16x8, prefetch 1 wins)
                zcs = ZCHUNKS or ((32,) if ty < 16 else (16,))
                for zc in zcs:
                    for pf in PREFETCH:
                        out.append(dict(tile_x=tx, tile_y=ty, threads=nt, block_x=bx, block_y=by,
                                        block_cby=cb, zchunk=zc, prefetch=pf))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--out", default=None)
    ap.add_argument("--top", type=int, default=8)
    ap.add_argument("--rounds", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--groups", default=None, help="comma list of group indices (default all)")
    ap.add_argument("--zchunks", default="", help="comma list of z-chunk lengths (default rule)")
    ap.add_argument("--prefetch", default="2,3", help="comma list of prefetch depths")
    a = ap.parse_args()
    global ZCHUNKS, PREFETCH
    ZCHUNKS = tuple(int(v) for v in a.zchunks.split(",") if v)
    PREFETCH = tuple(int(v) for v in a.prefetch.split(",") if v)
    prog = bench.load_workload(a.workload)
    plan = bench.plan_of(prog)
    cfgs = list(bench.tuned_configs(prog) or [None] * len(plan))
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream(dev)
    p = Program(prog)
    p.set_plan(plan)
    for i, c in enumerate(cfgs):
        if c:
            p.tune("fused", i, c)
    p.allocate(dev, fill=0.0)
    bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)

    def isolated(i, iters=7):
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
            ts.append(s.elapsed_time(e))
        return sorted(ts)[len(ts) // 2]

    def step_ms(reps=3):
        for _ in range(3):
            p.run_fused(stream)
        best = float("inf")
        for _ in range(reps):
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            torch.cuda.synchronize()
            s.record(stream)
            for _ in range(a.steps):
                p.run_fused(stream)
            e.record(stream)
            torch.cuda.synchronize()
            best = min(best, s.elapsed_time(e) / a.steps)
        return best

    def pin(i, c):
        p.tune("fused", i, c)

    t0 = time.time()
    base = step_ms()
    print(f"start: {base:.4f} ms/step", flush=True)
    groups = [int(g) for g in a.groups.split(",")] if a.groups else range(len(plan))
    for rnd in range(a.rounds):
        for i in groups:
            cur = cfgs[i]
            scored = []
            for c in candidates(prog["grid"]["ny"]):
                try:
                    pin(i, c)
                    scored.append((isolated(i), c))
                except StencilError:
                    continue
            scored.sort(key=lambda x: x[0])
            finalists = [c for _, c in scored[:a.top]]
            if cur is not None and cur not in finalists:
                finalists.append(cur)
            best_t, best_c = float("inf"), cur
            for c in finalists:
                try:
                    pin(i, c)
                except StencilError:
                    continue
                t = step_ms()
                if t < best_t:
                    best_t, best_c = t, c
            pin(i, best_c)
            cfgs[i] = best_c
            print(f"round {rnd} group {i}: {best_t:.4f} ms/step with {best_c} "
                  f"(isolated best {scored[0][0]*1e3:.1f} us; {len(scored)} candidates, "
                  f"{time.time()-t0:.0f} s)", flush=True)
    final = step_ms(reps=5)
    print(f"final: {final:.4f} ms/step (start {base:.4f})", flush=True)
    if a.out:
        src = os.environ.get("SF_C4_PLAN") or os.path.join(ROOT, "configs", "c4_plan.json")
        pj = json.load(open(src))
        pj["configs"] = cfgs
        pj["tuner"] = "tools/step_tune.py (in-context step timing)"
        pj["step_ms_tuned"] = final
        json.dump(pj, open(a.out, "w"), indent=1)
        print("wrote", a.out)


if __name__ == "__main__":
    main()
