"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE north star): inf-norm relative error <= 1e-12
(fp64) / 1e-5 (fp32) in the perf build (FMA contraction on); bit-exact against
the oracle and between fused and unfused with fmad=0 (the parity build:
same term order, no contraction, R4).  TEMP interiors are NaN-poisoned so a
fused kernel consuming a value it did not compute fails loudly.
"""
import json
import os

import numpy as np
import pytest

from _harness import assert_close, gpu_run, oracle_outputs, rel_err
from paper_conf_hpdc_wahibm15_b200 import StencilError
from synth import programs as P

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def closed_chain3_inputs(prog):
    g = prog["grid"]
    h = 1
    k, j, i = np.meshgrid(np.arange(-h, g["nz"] + h), np.arange(-h, g["ny"] + h),
                          np.arange(-h, g["nx"] + h), indexing="ij")
    f = {"A": i + 2.0 * j + 4 * k, "B": 1.0 + 0 * i, "T1": 2 * i + 4 * j + 8 * k + 1.0,
         "T2": 2 * i + 4 * j + 8 * k + 5.0, "O": 0.0 * i}
    out = {}
    for n, v in f.items():
        v = np.ascontiguousarray(v, dtype=np.float64)
        if n in ("T1", "T2", "O"):
            v[h:-h, h:-h, h:-h] = np.nan
        out[n] = v
    return out


@pytest.mark.parametrize("mode", ["unfused", "fused"])
@pytest.mark.parametrize("fmad", [0, 1])
def test_chain3_golden(cuda_device, mode, fmad):
    prog = P.chain3()
    gold = json.load(open(os.path.join(GOLDEN, "chain3.json")))
    got = gpu_run(prog, mode, 0, options={"fmad": fmad}, plan=prog["plans"]["fused"],
                  inputs=closed_chain3_inputs(prog))
    O = got["O"]
    for pt in gold["points"]:
        assert O[pt["k"], pt["j"], pt["i"]] == pt["O"]
    kk, jj, ii = np.meshgrid(np.arange(4), np.arange(4), np.arange(4), indexing="ij")
    assert np.array_equal(O, 1.5 * ii + 3 * jj + 6 * kk + 8.25)


CASES = [
    # (config builder, grid override, plan names)
    ("C1", P.c1(n=32), ["fused"]),
    ("C1odd", P.resize(P.c1(), 37, 11, 9), ["fused"]),
    ("C2", P.c2(nx=45, ny=37, nz=29), ["fused"]),
    ("C3", P.c3(nx=70, ny=41, nz=33), ["fused", "fission_fused", "single"]),
    ("C5", P.c5(nx=40, ny=23, nz=19), ["fused", "single"]),
    ("chain3", P.resize(P.chain3(), 33, 17, 13), ["fused"]),
]


@pytest.mark.parametrize("name,prog,plans", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("fmad", [0, 1])
def test_parity_vs_oracle(cuda_device, name, prog, plans, fmad):
    ref = oracle_outputs(prog, seed=11)
    exact = fmad == 0
    got = gpu_run(prog, "unfused", 11, options={"fmad": fmad})
    assert_close(prog, got, ref, exact=exact)
    for plan in plans:
        got = gpu_run(prog, "fused", 11, options={"fmad": fmad}, plan=prog["plans"][plan])
        assert_close(prog, got, ref, exact=exact)


# (tile, chunk, threads, prefetch, per-thread register block) combinations; the
# register block geometry fixes tile_y = (threads / (tile_x / block_x)) * block_y * block_cby
TILES = [dict(tile_x=16, tile_y=2, zchunk=1, threads=32, block_x=1, block_y=1, block_cby=1),
         dict(tile_x=32, tile_y=4, zchunk=3, threads=64, block_x=2, block_y=1, block_cby=1),
         dict(tile_x=64, tile_y=16, zchunk=7, threads=128, prefetch=1, block_x=2, block_y=2,
              block_cby=2),
         dict(tile_x=16, tile_y=16, zchunk=64, threads=64, prefetch=3, block_x=1, block_y=2,
              block_cby=2),
         dict(tile_x=64, tile_y=8, zchunk=5, threads=64, prefetch=2, block_x=4, block_y=2,
              block_cby=1)]


@pytest.mark.parametrize("tiles", TILES, ids=[str(i) for i in range(len(TILES))])
def test_tile_independence_bitexact(cuda_device, tiles):
    """Fused == unfused == oracle bit-exact with fmad=0 for any tile/chunk (P6)."""
    for prog, plan in [(P.c2(nx=37, ny=19, nz=17), "fused"),
                       (P.c3(nx=40, ny=21, nz=15), "fission_fused")]:
        ref = oracle_outputs(prog, seed=5)
        opts = dict(tiles, fmad=0)
        got = gpu_run(prog, "fused", 5, options=opts, plan=prog["plans"][plan])
        assert_close(prog, got, ref, exact=True)
        got = gpu_run(prog, "unfused", 5, options=opts)
        assert_close(prog, got, ref, exact=True)


@pytest.mark.parametrize("zqueue", [1, 2])
def test_zqueue_bitexact(cuda_device, zqueue):
    """Register z-queues (per statement / step-wide input columns) change no bit (P6)."""
    cases = [(P.c2(nx=37, ny=19, nz=17), "fused", (TILES[2], TILES[3])),
             (P.c3(nx=40, ny=21, nz=15), "fission_fused", (TILES[2], TILES[3])),
             (_c4_small(), "fused", ({}, dict(tile_x=32, tile_y=8, threads=64, block_x=1,
                                             block_y=4, block_cby=1, zchunk=5)))]
    for prog, plan, tile_set in cases:
        ref = oracle_outputs(prog, seed=6)
        for tiles in tile_set:
            opts = dict(tiles, fmad=0, zqueue=zqueue)
            got = gpu_run(prog, "fused", 6, options=opts, plan=prog["plans"][plan])
            assert_close(prog, got, ref, exact=True)
        got = gpu_run(prog, "unfused", 6, options={"fmad": 0, "zqueue": zqueue})
        assert_close(prog, got, ref, exact=True)


def test_c2_full_size(cuda_device):
    """BASELINE configs[1] at its full size (256^3 fp64), perf build, vs the oracle: the
    model-chosen tiles, then the bench's tuned per-launch configurations (fused and the
    tuned unfused baseline)."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    from _harness import gpu_program
    prog = P.c2()
    ref = oracle_outputs(prog, seed=2)
    for mode in ("unfused", "fused"):
        got = gpu_run(prog, mode, 2, plan=prog["plans"]["fused"])
        assert_close(prog, got, ref)
    bprog = bench.load_workload("C2")
    for mode in ("unfused", "fused"):
        p = gpu_program(bprog, plan=bprog["plans"]["fused"])
        bench.apply_tuning(p, bprog)
        got = gpu_run(bprog, mode, 2, program=p)
        assert_close(bprog, got, ref)


def _c4_small():
    import json as _json
    from synth.scale_les import c4
    prog = c4(nx=96, ny=32, nz=21)
    prog["plans"]["fused"] = _json.load(open(os.path.join(os.path.dirname(os.path.dirname(
        os.path.abspath(__file__))), "configs", "c4_plan.json")))["groups"]
    return prog


@pytest.mark.parametrize("mode", ["fused", "unfused"])
def test_c4_full_size_bench_configuration(cuda_device, mode):
    """BASELINE configs[3] at its full size (1280x32x256 fp64) in exactly the launch
    configuration bench.py times (frozen plan + tuned tiles, perf build; for "unfused"
    the tuned per-kernel configurations of the baseline the speedup is quoted against),
    against the full serial oracle (~5 s on the host)."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    from _harness import gpu_program
    prog = bench.load_workload("C4")
    ref = oracle_outputs(prog, seed=3)
    p = gpu_program(prog, plan=prog["plans"]["fused"])
    bench.apply_tuning(p, prog)
    got = gpu_run(prog, mode, 3, program=p)
    assert_close(prog, got, ref)


@pytest.mark.parametrize("fmad", [0, 1])
def test_c4_parity_reduced(cuda_device, fmad):
    """SCALE-LES-shaped 40-kernel DAG (BASELINE configs[3]) on a reduced grid, frozen greedy plan."""
    prog = _c4_small()
    ref = oracle_outputs(prog, seed=7)
    for mode in ("unfused", "fused"):
        got = gpu_run(prog, mode, 7, options={"fmad": fmad}, plan=prog["plans"]["fused"])
        assert_close(prog, got, ref, exact=(fmad == 0))


WAVES = [(1, 1), (3, 2), (5, 4), (8, 3), (16, 2)]


@pytest.mark.parametrize("zwave,streams", WAVES, ids=[f"S{a}x{b}" for a, b in WAVES])
def test_zwave_schedule_bitexact(cuda_device, zwave, streams):
    """z-wave schedule (launch i runs planes [wS - off_i, (w+1)S - off_i) per wave,
    waves in flight on several streams): bit-exact with the oracle (P6) for plans with
    RAW, WAR and WAW dependencies between groups, incl. tiny waves (S=1) that put
    every hazard distance at its minimum."""
    cases = [(P.c2(nx=37, ny=19, nz=17), ["fused"]),
             (P.c3(nx=40, ny=21, nz=23), ["fused", "fission_fused"]),
             (P.c5(nx=40, ny=23, nz=19), ["fused"]),
             (P.resize(P.chain3(), 33, 17, 13), ["fused"]),
             (_c4_small(), ["fused"])]
    for prog, plans in cases:
        ref = oracle_outputs(prog, seed=8)
        for plan in plans:
            opts = {"fmad": 0, "zwave": zwave, "zwave_streams": streams, "zchunk": 4}
            got = gpu_run(prog, "fused", 8, options=opts, plan=prog["plans"][plan], repeat=2)
            assert_close(prog, got, ref, exact=True)


def test_zwave_full_size_c4(cuda_device):
    """The bench's C4 launch configuration under the z-wave schedule, perf build, vs the
    plain plan order bit-exactly (same kernels, only the z-chunking differs)."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    from _harness import gpu_program
    prog = bench.load_workload("C4")
    outs = {}
    for zw in (0, 32):
        p = gpu_program(prog, options={"zwave": zw, "zwave_streams": 3},
                        plan=prog["plans"]["fused"])
        bench.apply_tuning(p, prog)
        outs[zw] = gpu_run(prog, "fused", 9, program=p, repeat=2)
    for n in outs[0]:
        assert outs[0][n].tobytes() == outs[32][n].tobytes(), n


@pytest.mark.parametrize("workload,plan,w", [("C5", "fused", 24), ("C3", "measured", 32),
                                             ("C3", "fission_fused", 32), ("C5", "unfused", 24),
                                             ("C3", "unfused", 32)])
def test_full_size_sampled_bench_configuration(cuda_device, workload, plan, w):
    """BASELINE configs[2] (C3, 512^3 fp32) and configs[4]'s per-GPU grid (C5, 1024x1024x128
    fp64) at full size, in the launch configuration bench.py times (plan + tuned tiles,
    perf build), checked on sampled windows the oracle evaluates one by one: corner,
    centre and far-corner windows of w^3 points; inside the window the oracle runs the
    whole program, and its result is exact wherever the window's margin covers the
    program's accumulated reach m (compared there; sides on the global boundary need no
    margin: their ghosts are the true ghosts, reading R1)."""
    import sys
    import torch
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    from _harness import accumulated_reach, gpu_program, rel_err, tolerance, window_field
    from oracle import OracleProgram
    prog = bench.load_workload(workload)
    g = prog["grid"]
    N = (g["nx"], g["ny"], g["nz"])
    h = tuple(g["ghost"])
    m = accumulated_reach(prog)
    unfused = plan == "unfused"  # the tuned unfused baseline (its configurations only)
    p = gpu_program(prog, plan=bench.plan_of(prog, "fused" if unfused else plan))
    bench.apply_tuning(p, prog, "fused" if unfused else plan)
    dev = torch.device("cuda:0")
    p.allocate(dev, fill=0.0)
    bench.fill_inputs(p, prog, dev, 0, h[2])
    p.run_unfused() if unfused else p.run_fused()
    torch.cuda.synchronize()
    outs = [a["name"] for a in prog["arrays"] if a["role"] in ("out", "inout")]
    orc = OracleProgram(prog)
    for origin in [(0, 0, 0), tuple((N[d] - w) // 2 for d in range(3)), tuple(N[d] - w for d in range(3))]:
        win = {a["name"]: window_field(4, aid, origin, (w, w, w), h, prog["dtype"])
               for aid, a in enumerate(prog["arrays"])}
        orc.run(win, n=(w, w, w), origin=origin)
        lo = [origin[d] + (m[d] if origin[d] > 0 else 0) for d in range(3)]
        hi = [origin[d] + w - (m[d] if origin[d] + w < N[d] else 0) for d in range(3)]
        assert all(hi[d] > lo[d] for d in range(3)), (lo, hi)
        for nm in outs:
            ref = win[nm][h[2] + lo[2] - origin[2]:h[2] + hi[2] - origin[2],
                          h[1] + lo[1] - origin[1]:h[1] + hi[1] - origin[1],
                          h[0] + lo[0] - origin[0]:h[0] + hi[0] - origin[0]]
            got = p.interior_view(p.tensors[nm])[lo[2]:hi[2], lo[1]:hi[1], lo[0]:hi[0]].cpu().numpy()
            e = rel_err(got, ref)
            assert e <= tolerance(prog["dtype"]), f"{workload} {nm} window {origin}: rel err {e}"


@pytest.mark.parametrize("mode", ["fused", "unfused"])
def test_cuda_graph_capture_replay_bitexact(cuda_device, mode):
    """S7: one step captured as a CUDA graph (torch.cuda.graph on its capture stream) and
    replayed equals the eagerly launched step bit for bit; replays are idempotent."""
    import sys
    import torch
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    from _harness import gpu_program
    prog = bench.load_workload("C4")
    prog = dict(prog, grid=dict(prog["grid"], nx=256, nz=64))
    p = gpu_program(prog, plan=prog["plans"]["fused"])
    dev = torch.device("cuda:0")
    p.allocate(dev, fill=0.0)
    bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
    outs = [a["name"] for a in prog["arrays"] if a["role"] in ("out", "inout")]
    p.run(mode)  # loads modules and builds launch parameters outside the capture
    torch.cuda.synchronize()
    want = {n: p.interior_view(p.tensors[n]).clone() for n in outs}
    for n in outs:
        p.interior_view(p.tensors[n]).fill_(float("nan"))
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream(device=dev)
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            p.run(mode, s)
    torch.cuda.synchronize()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    for n in outs:
        assert torch.equal(p.interior_view(p.tensors[n]), want[n]), f"{mode} {n}: graph replay differs"


@pytest.mark.parametrize("cfg", ["C3", "C4"])
def test_ga_plan_parity_bitexact(cuda_device, cfg):
    """Plans found by the GGA-lite search (sp_plan_search, NEXT #1) run bit-exact with
    the oracle in the parity build (fmad=0), fused and unfused."""
    from synth.scale_les import c4
    from paper_conf_hpdc_wahibm15_b200 import Program
    prog = {"C3": lambda: P.c3(nx=48, ny=20, nz=18), "C4": lambda: c4(nx=96, ny=32, nz=21)}[cfg]()
    plan = Program(prog).plan_search(generations=20, population=12, seed=5)
    ref = oracle_outputs(prog, seed=9)
    got = gpu_run(prog, "fused", 9, options={"fmad": 0}, plan=plan)
    assert_close(prog, got, ref, exact=True)


CLUSTER_CASES = [("C2", lambda: P.c2(nx=96, ny=24, nz=13), ["fused"]),
                 ("C3", lambda: P.c3(nx=128, ny=20, nz=11), ["fission_fused", "fused", "single"]),
                 ("C5", lambda: P.c5(nx=64, ny=17, nz=9), ["fused"]),
                 ("chain3", lambda: P.resize(P.chain3(), 70, 13, 9), ["fused"])]


@pytest.mark.parametrize("cx", [2, 4])
@pytest.mark.parametrize("name,mk,plans", CLUSTER_CASES, ids=[c[0] for c in CLUSTER_CASES])
def test_cluster_dsmem_halo_bitexact(cuda_device, name, mk, plans, cx):
    """Option cluster_x (NEXT #2): clusters of cx CTAs along x share the x-halo columns of
    shared-memory stages through DSMEM (remote mbarrier arrive + ld.shared::cluster) instead
    of recomputing them; fused == oracle bit-exact in the parity build, for tiles of 16
    and 32 columns (cluster edges inside and at the global x boundary), ragged grids."""
    from _harness import gpu_program
    prog = mk()
    ref = oracle_outputs(prog, seed=12)
    clustered = 0
    for tiles in ({}, dict(tile_x=16, tile_y=4, threads=64, block_x=1, block_y=1, block_cby=1, zchunk=4)):
        for plan in plans:
            p = gpu_program(prog, dict(tiles, fmad=0, cluster_x=cx), prog["plans"][plan])
            clustered += sum("constexpr int CX = %d;" % cx in l for l in p.source("fused").splitlines())
            got = gpu_run(prog, "fused", 12, program=p)
            assert_close(prog, got, ref, exact=True)
    assert clustered or cx == 4  # (a launch clusters only when its tile columns divide by cx)


DEGENERATE = [(1, 1, 1), (1, 7, 3), (5, 1, 1), (3, 2, 1), (2, 1, 9), (17, 1, 2)]


@pytest.mark.parametrize("n", DEGENERATE, ids=["x".join(map(str, n)) for n in DEGENERATE])
def test_degenerate_grids_bitexact(cuda_device, n):
    """Degenerate interiors (a single point, single rows / columns / planes): every ghost
    rule (R1) is in play at once, tiles are mostly outside the interior, z-chunks have one
    plane.  Unfused, fused (incl. fission + fusion) and a kernel with an EMPTY loop box
    (R2': writes nothing) in the parity build, bit-exact with the oracle."""
    cases = [(P.resize(P.c2(), *n), ["fused"]), (P.resize(P.c3(), *n), ["fused", "fission_fused"]),
             (P.resize(P.chain3(), *n), ["fused"])]
    boxed = P.resize(P.chain3(), *n)
    boxed["kernels"][1]["box"] = [0, 0, 0, n[1], 0, n[2]]  # empty in x: T2 keeps its stored value
    cases.append((boxed, ["fused"]))
    for prog, plans in cases:
        ref = oracle_outputs(prog, seed=13, poison=False)
        got = gpu_run(prog, "unfused", 13, options={"fmad": 0}, poison=False)
        assert_close(prog, got, ref, exact=True)
        for plan in plans:
            got = gpu_run(prog, "fused", 13, options={"fmad": 0}, plan=prog["plans"][plan], poison=False)
            assert_close(prog, got, ref, exact=True)


# Region-vector evaluation (option "frame"): every statement on its whole extended
# region in 16-byte x-vectors enumerated over the threads.  Tile shapes are free
# (tile_y independent of threads); ragged grids exercise edge tiles, partial last
# units (qq < nq) and ghost substitution on halo rows/columns left of / above the tile.
FRAME_TILES = [{}, dict(tile_x=16, tile_y=3, zchunk=2, threads=32),
               dict(tile_x=32, tile_y=16, zchunk=7, threads=128, prefetch=1, fastpath=1),
               dict(tile_x=64, tile_y=8, zchunk=5, threads=256, prefetch=2),
               dict(tile_x=32, tile_y=4, zchunk=9, threads=64, fastpath=1)]


@pytest.mark.parametrize("frame", [1, 2])
@pytest.mark.parametrize("name,prog,plans", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("fmad", [0, 1])
def test_frame_mode_parity(cuda_device, name, prog, plans, fmad, frame):
    """frame=1 / 2 (2: one unit grid per launch, own-position taps from register
    queues): fused plans (complex fusion with halo recompute, fission+fusion) match
    the oracle bit-exactly in the parity build and within R17 in the perf build."""
    ref = oracle_outputs(prog, seed=12)
    for tiles in FRAME_TILES:
        for plan in plans:
            try:
                got = gpu_run(prog, "fused", 12, options=dict(tiles, fmad=fmad, frame=frame),
                              plan=prog["plans"][plan])
            except StencilError as e:  # a pinned tile whose rings exceed shared memory
                assert tiles and e.code == 6, e
                continue
            assert_close(prog, got, ref, exact=fmad == 0)


def test_frame_mode_c4_reduced_bitexact(cuda_device):
    """frame=1 on the SCALE-LES-shaped 40-kernel DAG (reduced grid), bit-exact."""
    prog = _c4_small()
    ref = oracle_outputs(prog, seed=13)
    for tiles in ({}, dict(tile_x=32, tile_y=5, zchunk=4, threads=64)):
        for frame in (1, 2):
            got = gpu_run(prog, "fused", 13, options=dict(tiles, fmad=0, frame=frame),
                          plan=prog["plans"]["fused"])
            assert_close(prog, got, ref, exact=True)


@pytest.mark.parametrize("opts", [dict(rename=1), dict(rename=1, streams=2), dict(rename=1, streams=3),
                                  dict(streams=2), dict(rename=1, streams=2, frame=1)],
                         ids=["rename", "rename-s2", "rename-s3", "s2", "rename-s2-frame"])
def test_rename_and_dag_streams_bitexact(cuda_device, opts):
    """TEMP renaming (every later writer group of a TEMP stores into its own buffer
    instance, whose ghost cells are copied from the bound buffer) and the launch DAG on
    several streams (events between dependent launches) change no bit: every parity case
    and the 40-kernel C4 DAG (whose linear-scan TEMP reuse creates the WAR/WAW chains the
    renaming removes), fused, parity build, two steps (the second reuses the instances)."""
    cases = list(CASES) + [("C4small", _c4_small(), ["fused"])]
    for name, prog, plans in cases:
        ref = oracle_outputs(prog, seed=14)
        for plan in plans:
            got = gpu_run(prog, "fused", 14, options=dict(opts, fmad=0), plan=prog["plans"][plan])
            assert_close(prog, got, ref, exact=True)
        # two steps on the same program: OUT == oracle of two steps only for programs whose
        # OUT does not feed IN, so compare fused with the same program's unfused run instead
        p1 = gpu_run(prog, "fused", 14, options=dict(opts, fmad=0), plan=prog["plans"][plans[0]], repeat=2)
        p0 = gpu_run(prog, "fused", 14, options={"fmad": 0}, plan=prog["plans"][plans[0]], repeat=2)
        for n in p0:
            assert p1[n].tobytes() == p0[n].tobytes(), (name, n)


def test_dag_streams_graph_capture_bitexact(cuda_device):
    """The launch DAG on three streams captured into one CUDA graph (fork/join through
    events) and replayed: bit-identical to the eager single-stream step."""
    import torch
    from _harness import dense_arrays, gpu_program
    prog = _c4_small()
    arrs = dense_arrays(prog, 15, poison_temp=True)
    outs = {}
    for label, opts in (("eager", {}), ("graph", dict(rename=1, streams=3))):
        p = gpu_program(prog, dict(opts, fmad=0), prog["plans"]["fused"])
        dev = torch.device("cuda:0")
        p.allocate(dev)
        for n, d in arrs.items():
            p.padded_view(p.tensors[n]).copy_(torch.from_numpy(d))
        s = torch.cuda.Stream()
        if label == "graph":
            with torch.cuda.stream(s):
                p.run_fused(s)  # warm: shadows allocated and initialised outside the capture
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                p.run_fused(s)
            g.replay()
        else:
            p.run_fused(s)
        torch.cuda.synchronize()
        outs[label] = {a["name"]: p.interior_view(p.tensors[a["name"]]).cpu().numpy().copy()
                       for a in prog["arrays"] if a["role"] in ("out", "inout")}
    for n in outs["eager"]:
        assert outs["eager"][n].tobytes() == outs["graph"][n].tobytes(), n
