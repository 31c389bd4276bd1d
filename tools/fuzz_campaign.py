"""Long GPU fuzz campaign (dev tool; tests/test_gpu_fuzz.py runs a fixed 24-seed subset).

python tools/fuzz_campaign.py [--seeds 200] [--start 1000] [--ranks 0|2|3]

Single domain (--ranks 0): random programs (tests/_fuzz.py, half with loop bounds) under
the unfused plan and up to four accepted fusion plans, with random tile / chunk / block
options, parity build, bit-exact against the oracle.  Multi-rank (--ranks P): the same
programs on P loopback virtual ranks (z-slabs with deep halos, the executor's exchange
schedule and interior/boundary split), two steps, bit-exact against the single domain.
Prints one line per failure and a summary.
"""
import argparse
import os
import sys
import threading
import traceback

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

TILES = [{}, dict(tile_x=16, tile_y=2, threads=32, block_x=1, block_y=1, block_cby=1, zchunk=1),
         dict(tile_x=32, tile_y=4, threads=64, block_x=2, block_y=1, block_cby=1, zchunk=3),
         dict(tile_x=16, tile_y=16, threads=64, block_x=1, block_y=2, block_cby=2, zchunk=5, prefetch=3),
         dict(tile_x=64, tile_y=8, threads=64, block_x=4, block_y=2, block_cby=1, zchunk=2, prefetch=2)]


# region-vector (frame) evaluation: tile_y is free of the thread count
FRAME_TILES = [dict(frame=1), dict(frame=1, tile_x=16, tile_y=3, threads=32, zchunk=2),
               dict(frame=1, tile_x=32, tile_y=5, threads=64, zchunk=3, fastpath=1),
               dict(frame=1, tile_x=64, tile_y=8, threads=256, zchunk=4, prefetch=2)]


def single(seed, boxes, frame=False):
    from _fuzz import fuzz_case
    from _harness import assert_close, gpu_run, oracle_outputs
    prog, plans, _, _ = fuzz_case(seed, boxes)
    rng = np.random.default_rng(seed)
    ref = oracle_outputs(prog, seed=seed, poison=False)
    tiles = FRAME_TILES if frame else TILES
    opts = dict(tiles[int(rng.integers(0, len(tiles)))], fmad=0)
    if frame:
        opts["frame"] = frame
        if boxes:  # loop-bounded groups keep the block form: no frame-only (free tile_y) shapes
            opts = {"fmad": 0, "frame": frame}
    # frame shapes (free tile_y) apply to fused groups; the unfused kernels keep the block form
    uopts = {"fmad": 0} if frame else opts
    assert_close(prog, gpu_run(prog, "unfused", seed, options=uopts, poison=False), ref, exact=True)
    from paper_conf_hpdc_wahibm15_b200 import StencilError
    for plan in plans:
        try:
            got = gpu_run(prog, "fused", seed, options=opts, plan=plan, poison=False)
        except StencilError as e:  # a pinned frame shape whose rings do not fit this group
            if e.code == 6 and frame and "tile_x" in opts:
                continue
            raise
        assert_close(prog, got, ref, exact=True)


def multi(seed, boxes, ranks):
    import torch
    from _fuzz import fuzz_case
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    from test_gpu_multirank import fill
    prog, plans, _, _ = fuzz_case(seed, boxes)
    g = prog["grid"]
    nzl = max(12, g["nz"])
    dev = torch.device("cuda:0")

    def with_nz(nz):
        q = dict(prog, grid=dict(g, nz=nz))
        for k in q["kernels"]:  # boxes are in global coordinates: keep them inside the grid
            if k.get("box") is not None:
                b = list(k["box"])
                b[5] = min(b[5], nz)
                b[4] = min(b[4], b[5])
                k["box"] = b
        return q
    glob = with_nz(nzl * ranks)
    loc = with_nz(nzl)
    loc["kernels"] = glob["kernels"]
    for plan in [None] + plans[:2]:
        mode = "unfused" if plan is None else "fused"
        single_p = Program(glob, options={"fmad": 0})
        if plan:
            single_p.set_plan(plan)
        single_p.allocate(dev)
        fill(single_p, glob, dev, 0, g["ghost"][2])
        for _ in range(2):
            single_p.run(mode)
        probe = Program(loc, nz_global=nzl * ranks)
        if plan:
            probe.set_plan(plan)
        zhalo = max([max(r["z_below"], r["z_above"]) for m in (["fused"] if plan else []) + ["unfused"]
                     for r in probe.reports(m)] + [g["ghost"][2]])
        comms = Comm.loopback(ranks)
        slabs = []
        for r in range(ranks):
            s = Program(loc, comm=comms[r], nz_global=nzl * ranks, z_offset=r * nzl, zhalo=zhalo,
                        options={"fmad": 0})
            if plan:
                s.set_plan(plan)
            s.allocate(dev)
            fill(s, loc, dev, r * nzl, zhalo, nz_global=nzl * ranks)
            s.load(mode)
            slabs.append(s)
        torch.cuda.synchronize()
        errs = []

        def drive(r):
            try:
                st = torch.cuda.Stream(device=dev)
                for _ in range(2):
                    slabs[r].run(mode, st)
                st.synchronize()
            except Exception as e:  # noqa: BLE001
                errs.append(e)
        th = [threading.Thread(target=drive, args=(r,)) for r in range(ranks)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        assert not errs, errs
        torch.cuda.synchronize()
        for a in prog["arrays"]:
            if a["role"] not in ("out", "inout"):
                continue
            n = a["name"]
            want = single_p.interior_view(single_p.tensors[n])
            got = torch.cat([s.interior_view(s.tensors[n]) for s in slabs], dim=0)
            assert torch.equal(got.nan_to_num(123.0), want.nan_to_num(123.0)), f"{mode} {plan}: {n} differs"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, default=200)
    ap.add_argument("--start", type=int, default=1000)
    ap.add_argument("--ranks", type=int, default=0)
    ap.add_argument("--frame", type=int, default=0, help="fused plans in region-vector (frame) mode 1 / 2")
    a = ap.parse_args()
    fails = 0
    for seed in range(a.start, a.start + a.seeds):
        for boxes in (False, True):
            try:
                if a.ranks:
                    multi(seed, boxes, a.ranks)
                else:
                    single(seed, boxes, a.frame)
            except Exception:  # noqa: BLE001
                fails += 1
                print(f"FAIL seed {seed} boxes {boxes}: {traceback.format_exc().splitlines()[-1][:300]}",
                      flush=True)
    print(f"fuzz campaign ranks={a.ranks} frame={int(a.frame)}: {2 * a.seeds} cases, {fails} failures",
          flush=True)


if __name__ == "__main__":
    main()
