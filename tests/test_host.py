"""Host-side logic of the library (no GPU): C-ABI exports, program validation,
DDG/OEG edges, fission (Algorithm 2), plan legality, group analysis, the
byte/flop model and NVRTC compilation of the generated sm_100a kernels."""
import ctypes
import os
import re

import pytest

from paper_conf_hpdc_wahibm15_b200 import Program, StencilError
from paper_conf_hpdc_wahibm15_b200._abi import EXPORTS, LIB_PATH
from synth import programs as P

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

pytestmark = pytest.mark.host

HEADER = "include/stencilfuse.h"


def test_library_exports_every_header_symbol():
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    text = open(os.path.join(root, HEADER)).read()
    declared = set(re.findall(r"^\s*(?:sp_status|void|const char \*)\s*\*?\s*(\w+)\s*\(", text, re.M))
    assert declared == set(EXPORTS), declared ^ set(EXPORTS)
    lib = ctypes.CDLL(LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name


def test_no_gpu_run_fails_loudly_without_device():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    p = Program(P.c1(n=8))
    with pytest.raises(StencilError) as e:
        p.run_unfused(stream=0)
    assert e.value.code in (8, 10)  # SP_E_CUDA (no device) / SP_E_STATE (unbound)


# ----------------------------------------------------------------- validation
def bad(prog):
    with pytest.raises(StencilError) as e:
        Program(prog)
    return e.value.code


def test_rejects_r3_in_kernel_race():
    prog = P.c1(n=8)
    prog["kernels"] = [P.kernel("K", P.stmt("T", [{"c": 1.0, "a": ["A", 0, 0, 0]}]),
                                P.stmt("B", [{"c": 1.0, "a": ["T", 0, 1, 0]}]))]
    assert bad(prog) == 2


def test_rejects_tap_beyond_ghost():
    prog = P.c1(n=8)
    prog["kernels"] = [P.kernel("K", P.stmt("T", [{"c": 1.0, "a": ["A", 0, 0, 2]}]))]
    assert bad(prog) == 2


def test_rejects_write_to_input():
    prog = P.c1(n=8)
    prog["kernels"] = [P.kernel("K", P.stmt("A", [{"c": 1.0, "a": ["T", 0, 0, 0]}]))]
    assert bad(prog) == 2


def test_layout_alignment():
    for prog in (P.c1(n=33), P.c3(n=17)):
        p = Program(prog)
        L = p.layout
        assert (L["x_pitch"] * p.elem) % 128 == 0
        assert (L["origin_x"] * p.elem) % 128 == 0
        assert L["origin_x"] >= p.ghost[0] and L["x_pitch"] >= L["origin_x"] + p.n[0] + p.ghost[0]
        assert L["bytes"] == L["x_pitch"] * L["y_alloc"] * L["z_alloc"] * p.elem


# ----------------------------------------------------------------- DDG / OEG
def test_edges_c2():
    p = Program(P.c2(n=8))
    e = {(a, b): k for a, b, k, _ in p.edges()}
    # stmt ids: grad 0,1,2; flux 3,4,5; div 6; update 7
    assert e[(0, 3)] & 1 and e[(1, 4)] & 1 and e[(2, 5)] & 1      # RAW g -> F
    assert e[(3, 6)] & 1 and e[(6, 7)] & 1                         # RAW F -> D -> phin
    assert (0, 1) not in e and (3, 4) not in e                     # independent siblings


def test_edges_war_waw_c5_temp_reuse():
    p = Program(P.c5(nx=8, ny=8, nz=8))
    kinds = {}
    for a, b, k, arr in p.edges():
        kinds[(a, b)] = k
    # tracer 1's gradient (stmt 8) rewrites gx (stmt 0 wrote it, stmt 3 read it)
    assert kinds[(0, 8)] & 4          # WAW
    assert kinds[(3, 8)] & 2          # WAR


# ----------------------------------------------------------------- fission
def fig3_program():
    """Reconstruction of Fig. 3's Kern_A (garbled): R, W <- S, V and
    T, U <- Q, P; after fission Kern_X keeps R, W with S, V."""
    arr = [(n, "in") for n in "SVQP"] + [(n, "out") for n in "RWTU"]
    st = lambda o, a, b: P.stmt(o, [{"c": 1.0, "a": [a, 0, 0, 0]}, {"c": 0.5, "a": [b, 1, 0, 0]}])
    return {"name": "fig3", "dtype": "f64", "grid": {"nx": 8, "ny": 8, "nz": 8, "ghost": [1, 1, 1]},
            "arrays": [{"name": n, "role": r} for n, r in arr],
            "kernels": [P.kernel("Kern_A", st("R", "S", "V"), st("T", "Q", "P"), st("W", "S", "V"),
                                 st("U", "P", "Q"))]}


def test_fission_fig3():
    p = Program(fig3_program())
    comp, n = p.fission("Kern_A")
    assert n == 2
    assert comp == [0, 1, 0, 1]  # {R, W} and {T, U}, ordered by first statement


def test_fission_c3_k0_separable_and_shared_input_stays():
    p = Program(P.c3(n=8))
    assert p.fission("K0") == ([0, 1], 2)
    prog = P.c3(n=8)
    prog["kernels"][0]["stmts"][1]["terms"].append({"c": 1.0, "a": ["A", 0, 0, 0]})
    assert Program(prog).fission("K0") == ([0, 0], 1)  # shared input A joins the pieces


# ----------------------------------------------------------------- plan legality
def test_plan_partition_errors():
    prog = P.c2(n=8)
    p = Program(prog)
    with pytest.raises(StencilError) as e:
        p.set_plan([["grad", "flux"], ["div"]])            # update missing
    assert e.value.code == 3
    with pytest.raises(StencilError) as e:
        p.set_plan([["grad", "flux"], ["flux:0", "div", "update"]])  # twice
    assert e.value.code == 3


def test_plan_order_error():
    p = Program(P.c2(n=8))
    with pytest.raises(StencilError) as e:
        p.set_plan([["flux", "div", "update"], ["grad"]])
    assert e.value.code == 4


def test_plan_hazard_war_in_group():
    """K1 reads A at +x, K2 writes A (stored for a later group): SP_E_PLAN_HAZARD (R11)."""
    prog = {"name": "war", "dtype": "f64", "grid": {"nx": 16, "ny": 8, "nz": 8, "ghost": [1, 1, 1]},
            "arrays": [{"name": "A", "role": "inout"}, {"name": "X", "role": "in"},
                       {"name": "T", "role": "out"}],
            "kernels": [P.kernel("K1", P.stmt("T", [{"c": 0.5, "a": ["A", 1, 0, 0]}])),
                        P.kernel("K2", P.stmt("A", [{"c": 2.0, "a": ["X", 0, 0, 0]}]))]}
    p = Program(prog)
    with pytest.raises(StencilError) as e:
        p.set_plan([["K1", "K2"]])
    assert e.value.code == 5
    p.set_plan([["K1"], ["K2"]])  # split: legal
    # point-wise read of the own tile before the store is the allowed exception
    prog["kernels"][0]["stmts"][0]["terms"][0]["a"] = ["A", 0, 0, 0]
    Program(prog).set_plan([["K1", "K2"]])


def test_failed_plan_keeps_previous():
    p = Program(P.c2(n=8))
    p.set_plan([["grad", "flux", "div", "update"]])
    with pytest.raises(StencilError):
        p.set_plan([["update"], ["grad", "flux", "div"]])
    assert p.n_launches("fused") == 1


# ----------------------------------------------------------------- analysis / model
def passes(p, mode):
    return sum(r["bytes_alg"] for r in p.reports(mode)) / p.elem


def test_bytes_model_c2():
    """C2: unfused 21 passes -> fused 5 (pin P10)."""
    prog = P.c2(n=64)
    p = Program(prog)
    assert passes(p, "unfused") == 21
    p.set_plan(prog["plans"]["fused"])
    assert passes(p, "fused") == 5
    r = p.reports("fused")[0]
    assert r["n_inputs"] == 4 and r["n_stores"] == 1


def test_bytes_model_c3():
    """C3: 21 -> 8 (no fission) -> 5 (fission + fusion) -> 3 (single group)."""
    prog = P.c3(n=64)
    p = Program(prog)
    assert passes(p, "unfused") == 21
    for plan, want in (("fused", 8), ("fission_fused", 5), ("single", 3)):
        p.set_plan(prog["plans"][plan])
        assert passes(p, "fused") == want, plan


def test_group_analysis_c2_appendix_b():
    """Per-statement extension/lead/storage of C2's fused group."""
    prog = P.c2(n=64)
    p = Program(prog)
    p.set_plan(prog["plans"]["fused"])
    src = p.source("fused")
    info = {}
    for m in re.finditer(r"// stmt (\S+) -> (\S+)\s+lead (-?\d+), planes \[(-?\d+), zc-1\+(-?\d+)\], "
                         r"ext \((-?\d+),(-?\d+),(-?\d+),(-?\d+)\)(, stored)?, (register|smem ring) "
                         r"depth (\d+)", src):
        info[m.group(2)] = dict(lead=int(m.group(3)), ext=tuple(int(m.group(i)) for i in range(6, 10)),
                                stored=bool(m.group(10)), keep=m.group(11), depth=int(m.group(12)))
    assert info["phin"] == dict(lead=0, ext=(0, 0, 0, 0), stored=True, keep="register", depth=1)
    assert info["D"]["ext"] == (0, 0, 0, 0) and info["D"]["keep"] == "register"
    assert info["Fx"]["ext"] == (1, 1, 0, 0) and info["Fx"]["keep"] == "smem ring"
    assert info["Fy"]["ext"] == (0, 0, 1, 1) and info["Fy"]["keep"] == "smem ring"
    assert info["Fz"] == dict(lead=1, ext=(0, 0, 0, 0), stored=False, keep="register", depth=3)
    assert info["gx"]["ext"] == (1, 1, 0, 0) and info["gx"]["keep"] == "register"
    assert info["gz"]["lead"] == 1 and info["gz"]["keep"] == "register"


def test_group_analysis_chain3():
    prog = P.chain3()
    p = Program(prog)
    p.set_plan(prog["plans"]["fused"])
    src = p.source("fused")
    assert re.search(r"-> T2\s+lead 1, planes \[0, zc-1\+1\], ext \(1,0,0,0\)", src)
    assert re.search(r"-> T1\s+lead 1, planes \[0, zc-1\+1\], ext \(1,0,1,0\)", src)


def test_dead_statement_skipped():
    """A TEMP overwritten before any read inside the group is never computed."""
    prog = {"name": "dead", "dtype": "f64", "grid": {"nx": 16, "ny": 8, "nz": 8, "ghost": [1, 1, 1]},
            "arrays": [{"name": "X", "role": "in"}, {"name": "T", "role": "temp"},
                       {"name": "Y", "role": "out"}],
            "kernels": [P.kernel("K1", P.stmt("T", [{"c": 3.0, "a": ["X", 1, 0, 0]}])),
                        P.kernel("K2", P.stmt("T", [{"c": 2.0, "a": ["X", 0, 0, 0]}])),
                        P.kernel("K3", P.stmt("Y", [{"c": 1.0, "a": ["T", 0, 0, 1]}]))]}
    p = Program(prog)
    p.set_plan([["K1", "K2", "K3"]])
    assert p.reports("fused")[0]["n_stmts"] == 2


# ----------------------------------------------------------------- NVRTC (sm_100a) compile
@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C5", "chain3"])
def test_generated_kernels_compile_for_sm100a(name):
    prog = P.chain3() if name == "chain3" else P.CONFIGS[name]()
    for fmad in (0, 1):
        p = Program(prog, options={"fmad": fmad})
        p.compile("unfused")
        for plan_name, plan in prog["plans"].items():
            if plan_name == "unfused":
                continue
            p.set_plan(plan)
            p.compile("fused")
            for r in p.reports("fused"):
                assert 0 < r["regs_per_thread"] <= 255
                assert r["smem_bytes"] <= 227 * 1024


# ----------------------------------------------------------------- tuning / exchange / planner
def test_plan_tune_pins_and_resets():
    prog = P.c2(n=64)
    p = Program(prog)
    p.set_plan(prog["plans"]["fused"])
    cfg = dict(tile_x=64, tile_y=8, threads=128, block_x=1, block_y=4, block_cby=1, zchunk=16)
    p.tune("fused", 0, cfg)
    r = p.report("fused", 0)
    assert (r["tile_x"], r["tile_y"], r["threads"], r["block_y"], r["zchunk"]) == (64, 8, 128, 4, 16)
    p.tune("fused", 0, None)
    assert p.report("fused", 0)["tile_y"] != 8 or p.report("fused", 0)["zchunk"] != 16
    with pytest.raises(StencilError) as e:   # inconsistent thread geometry
        p.tune("fused", 0, dict(tile_x=64, tile_y=3, threads=128, block_x=1, block_y=1, block_cby=1))
    assert e.value.code == 6
    p.tune("fused", 0, cfg)
    p.set_plan(prog["plans"]["fused"])      # a new plan drops the pins
    assert p.report("fused", 0)["zchunk"] != 16 or p.report("fused", 0)["tile_y"] != 8


def test_exchange_schedule_matches_reach():
    prog = P.c3(n=32)
    p = Program(prog, nz_global=64, z_offset=0, zhalo=5)
    p.set_plan(prog["plans"]["fission_fused"])
    # IN arrays (step-start epochs) all travel in one exchange in front of the first launch;
    # 7pt, 7pt, 13pt, 7pt chain: reach 1+1+2+1
    assert p.exchange_plan("fused", 0) == [("A", 5, 5), ("B", 5, 5)]
    assert p.exchange_plan("fused", 1) == []
    # unfused: each array once per epoch (after its writer), before its first halo reader
    want = {0: [("A", 1, 1), ("B", 1, 1)], 1: [("P", 1, 1)], 2: [("P1", 2, 2)], 3: [("P2", 1, 1)],
            4: [("Q", 1, 1)], 5: [("Q1", 2, 2)], 6: [("Q2", 1, 1)], 7: []}
    assert {i: p.exchange_plan("unfused", i) for i in range(8)} == want


def test_exchange_schedule_hoists_unchanged_arrays():
    """An array read beyond the slab by several launches between two writes is received
    once, before the first of them, at the largest depth any of them needs (C4)."""
    from synth.scale_les import c4
    prog = c4(nx=64, ny=32, nz=32)
    p = Program(prog, nz_global=64, z_offset=0, zhalo=4)
    names = [a["name"] for a in prog["arrays"]]
    n = p.n_launches("unfused")
    got = {i: p.exchange_plan("unfused", i) for i in range(n)}
    # replay: every halo read of every launch is covered by the last reception of that
    # array since its last store, and nothing is received twice inside one epoch
    fresh = {}
    for i in range(n):
        for a, lo, hi in got[i]:
            assert a not in fresh, f"{a} received twice in one epoch"
            fresh[a] = (lo, hi)
        r = p.report("unfused", i)
        k = prog["kernels"][i]
        for st in k["stmts"]:
            for t in st["terms"]:
                for tap in ([t["a"]] + ([t["b"]] if t.get("b") else [])):
                    arr, dz = tap[0], tap[3]
                    if dz:
                        lo, hi = fresh[arr]
                        assert (-dz <= lo) if dz < 0 else (dz <= hi), (i, arr, dz)
        for st in k["stmts"]:
            fresh.pop(st["out"], None)
    assert sum(len(v) for v in got.values()) < sum(
        1 for k in prog["kernels"] for st in k["stmts"] for t in st["terms"])


def test_deep_halo_must_cover_reach():
    prog = P.c3(n=32)
    p = Program(prog, nz_global=64, z_offset=0, zhalo=4)
    p.set_plan(prog["plans"]["unfused"])          # reach <= 2: fine
    # single-rank programs do not exchange, so any reach is allowed there
    q = Program(prog, zhalo=2)
    q.set_plan(prog["plans"]["single"])


def test_greedy_plan_is_legal_and_reduces_traffic():
    from synth.scale_les import c4
    prog = c4(nx=256, ny=32, nz=64)
    p = Program(prog)
    plan = p.plan_greedy()
    p.set_plan(plan)
    fused = sum(r["bytes_alg"] for r in p.reports("fused"))
    unfused = sum(r["bytes_alg"] for r in p.reports("unfused"))
    assert fused < 0.7 * unfused
    refs = [r for g in plan for r in g]
    assert len(refs) == len(set(refs)) == sum(len(k["stmts"]) for k in prog["kernels"])


def _model_cost(p, plan):
    p.set_plan(plan)
    return sum(r["t_model_us"] for r in p.reports("fused"))


@pytest.mark.parametrize("cfg", ["C3", "C4", "fuzz"])
def test_ga_plan_search_legal_deterministic_not_worse(cfg):
    """GGA-lite (sp_plan_search, NEXT #1): the plan is a legal partition accepted by
    fusion_plan_set, identical for the same seed, and its modelled step time is not
    above the greedy plan's (the GA is seeded with it; elitism)."""
    import numpy as np
    from synth.scale_les import c4
    from _fuzz import random_lib_program
    prog = {"C3": lambda: P.c3(n=64), "C4": lambda: c4(nx=256, ny=32, nz=64),
            "fuzz": lambda: random_lib_program(np.random.default_rng(3))}[cfg]()
    p = Program(prog)
    g = p.plan_greedy()
    s1 = p.plan_search(generations=25, population=12, seed=7)
    assert s1 == p.plan_search(generations=25, population=12, seed=7)
    refs = [r for grp in s1 for r in grp]
    assert len(refs) == len(set(refs)) == sum(len(k["stmts"]) for k in prog["kernels"])
    assert _model_cost(p, s1) <= _model_cost(p, g) * 1.02   # full vs quick tile search


def test_ga_plan_search_interleaved_chains():
    """Two independent chains interleaved in program order (A1, B1, A2, B2): the search
    (whose decoding may group independent units out of program order) returns a legal
    plan that moves each array once (no temp round trip)."""
    T = P.tap
    prog = {"name": "interleaved", "dtype": "f64", "grid": {"nx": 64, "ny": 32, "nz": 32, "ghost": [1, 1, 1]},
            "arrays": [{"name": n, "role": r} for n, r in
                       (("A", "in"), ("B", "in"), ("X", "temp"), ("Y", "temp"), ("OA", "out"), ("OB", "out"))],
            "kernels": [P.kernel("A1", P.stmt("X", P.stencil_terms("A", P.PT7, [1 / 7] * 7))),
                        P.kernel("B1", P.stmt("Y", P.stencil_terms("B", P.PT7, [1 / 7] * 7))),
                        P.kernel("A2", P.stmt("OA", [{"c": 0.5, "a": T("X", (0, 0, 0))}])),
                        P.kernel("B2", P.stmt("OB", [{"c": 0.5, "a": T("Y", (0, 0, 0))}]))]}
    p = Program(prog)
    s = p.plan_search(generations=30, population=16, seed=1)
    p.set_plan(s)
    assert _model_cost(p, s) <= _model_cost(p, p.plan_greedy()) * 1.02
    fused = sum(r["bytes_alg"] for r in p.reports("fused"))
    assert fused <= 4 * 8  # A, B, OA, OB once each


def test_wave_offsets_raw_reach():
    """z-wave skew: K3 reads T2 one plane above (dz=+1), so it trails K2 by one plane;
    point-wise and in-plane reads need no skew."""
    prog = P.resize(P.chain3(), 16, 8, 12)
    p = Program(prog)
    p.set_plan([["K1"], ["K2"], ["K3"]])
    assert p.wave_offsets() == [0, 0, 1]
    p.set_plan(prog["plans"]["fused"])
    assert p.wave_offsets() == [0]


def test_wave_offsets_war_waw():
    """WAR: K2 overwrites X, which K1 reads two planes below, so K2 trails K1 by 2;
    K3 reads K2's X point-wise (RAW, no reach) and inherits the skew."""
    T = P.tap
    prog = {"name": "war", "dtype": "f64", "grid": {"nx": 16, "ny": 8, "nz": 12, "ghost": [1, 1, 2]},
            "arrays": [{"name": n, "role": r} for n, r in
                       (("A", "in"), ("B", "in"), ("X", "temp"), ("Y", "temp"), ("O", "out"))],
            "kernels": [P.kernel("K0", P.stmt("X", [{"c": 1.0, "a": T("A", (0, 0, 0))}])),
                        P.kernel("K1", P.stmt("Y", [{"c": 1.0, "a": T("X", (0, 0, -2))}])),
                        P.kernel("K2", P.stmt("X", [{"c": 1.0, "a": T("B", (0, 0, 0))}])),
                        P.kernel("K3", P.stmt("O", [{"c": 1.0, "a": T("Y", (0, 0, 0))},
                                                    {"c": 1.0, "a": T("X", (0, 0, 0))}]))]}
    p = Program(prog)
    p.set_plan([["K0"], ["K1"], ["K2"], ["K3"]])
    assert p.wave_offsets() == [0, 0, 2, 2]


def test_fuzz_plans_legal_or_rejected_and_compile():
    """Random legal programs (with and without loop bounds, R2') and random plans:
    set_plan either accepts the plan or raises a plan error (never another failure),
    and every accepted plan's kernels compile for sm_100a (NVRTC, no GPU needed)."""
    import numpy as np
    from _fuzz import random_lib_program, random_plans
    accepted = rejected = 0
    for seed in range(6):
        rng = np.random.default_rng(seed)
        prog = random_lib_program(rng, boxes=bool(seed % 2))
        p = Program(prog)
        p.compile("unfused")
        for plan in random_plans(rng, prog, count=2):
            try:
                p.set_plan(plan)
            except StencilError as e:
                assert e.code in (4, 5, 6), e   # SP_E_PLAN_ORDER / _HAZARD / SP_E_RESOURCES
                rejected += 1
                continue
            p.compile("fused")
            accepted += 1
    assert accepted > 0


def test_box_validation_and_hazard():
    T = P.tap
    base = {"name": "b", "dtype": "f64", "grid": {"nx": 8, "ny": 6, "nz": 5, "ghost": [1, 1, 1]},
            "arrays": [{"name": "A", "role": "in"}, {"name": "X", "role": "temp"},
                       {"name": "O", "role": "out"}]}
    k0 = {"name": "K0", "stmts": [{"out": "X", "terms": [{"c": 1.0, "a": T("A", (0, 0, 0))}]}]}
    k1 = {"name": "K1", "box": [0, 8, 0, 6, 0, 1],
          "stmts": [{"out": "X", "terms": [{"c": 2.0, "a": T("A", (0, 0, 1))}]}]}
    k2 = {"name": "K2", "stmts": [{"out": "O", "terms": [{"c": 1.0, "a": T("X", (1, 0, 0))}]}]}
    bad = dict(base, kernels=[dict(k1, box=[0, 9, 0, 6, 0, 1])])
    with pytest.raises(StencilError) as e:
        Program(bad)
    assert e.value.code == 2                           # SP_E_PROGRAM: box beyond the interior
    p = Program(dict(base, kernels=[k0, k1, k2]))
    with pytest.raises(StencilError) as e:             # K0 and boxed K1 both write X in a group
        p.set_plan([["K0", "K1", "K2"]])
    assert "R2'" in str(e.value)
    p.set_plan([["K0"], ["K1", "K2"]])                 # boxed writer alone in its group: fine
    p.compile("fused")


def test_segment_dp_is_exact():
    """The measured planner's segmentation DP (tools/plan_autotune.py, NEXT #1) returns
    the optimum over contiguous segmentations, checked by brute force on random costs
    (including illegal segments)."""
    import itertools
    import os
    import sys
    import numpy as np
    sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
    import importlib
    pa = importlib.import_module("plan_autotune")
    rng = np.random.default_rng(0)
    for n, mu in ((6, 3), (7, 7), (8, 2)):
        c = {(i, j): (float("inf") if rng.random() < 0.15 and j - i > 1 else float(rng.random() * (j - i) ** 0.7))
             for i in range(n) for j in range(i + 1, n + 1)}
        cuts = pa.segment_dp(n, lambda i, j: c[(i, j)], mu)
        got = sum(c[(a, b)] for a, b in zip(cuts[:-1], cuts[1:]))
        best = float("inf")
        for mask in itertools.product([0, 1], repeat=n - 1):
            cs = [0] + [i + 1 for i, m in enumerate(mask) if m] + [n]
            if any(b - a > mu for a, b in zip(cs[:-1], cs[1:])):
                continue
            best = min(best, sum(c[(a, b)] for a, b in zip(cs[:-1], cs[1:])))
        assert abs(got - best) < 1e-12 and all(b - a <= mu for a, b in zip(cuts[:-1], cuts[1:]))


@pytest.mark.parametrize("mode", ["fused", "unfused"])
def test_peer_push_schedule_and_codegen(mode):
    """NEXT #2 host side (no GPU): with option xpush on a 2-rank communicator, every TEMP
    epoch that begins at a store leaves the communicator's schedule (its storing kernel
    pushes it), step-start epochs stay, the generated kernels carry the push stores and
    the progress protocol, and they compile for sm_100a (NVRTC)."""
    from synth.scale_les import c4
    from paper_conf_hpdc_wahibm15_b200 import Comm
    import json
    import os
    prog = c4(nx=64, ny=32, nz=16)
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    prog["plans"]["fused"] = json.load(open(os.path.join(root, "configs", "c4_plan.json")))["groups"]
    temps = {a["name"] for a in prog["arrays"] if a["role"] == "temp"}
    comms = Comm.loopback(2)
    p = Program(prog, comm=comms[0], nz_global=32, z_offset=0, zhalo=4, options={"xpush": 1})
    q = Program(prog, comm=comms[1], nz_global=32, z_offset=16, zhalo=4)
    for x in (p, q):
        x.set_plan(prog["plans"]["fused"])
    n = p.n_launches(mode)
    with_push = [p.exchange_plan(mode, i) for i in range(n)]
    without = [q.exchange_plan(mode, i) for i in range(n)]
    assert not any(a in temps for x in with_push for a, _, _ in x)
    assert with_push[0] == without[0]                       # step-start epochs unchanged
    assert any(a in temps for x in without for a, _, _ in x)  # TEMP epochs did travel before
    src = p.source(mode)
    assert "push down" in src and "push up" in src and "sf_xs_wait" in src and "sf_xs_signal" in src
    assert "push down" not in q.source(mode)
    p.compile(mode)


def test_fuzz_cases_run_fused_plans():
    """Every GPU fuzz case (tests/test_gpu_fuzz.py) has >= 2 accepted fusion plans; boxed
    cases fuse a boxed kernel with another statement (R2'); rejected candidates carry a
    plan error (SP_E_PLAN_ORDER / _HAZARD / _RESOURCES)."""
    from _fuzz import _fuses_boxed, fuzz_case
    for boxes in (False, True):
        for seed in range(12):
            prog, plans, rejected, _ = fuzz_case(seed, boxes)
            assert len(plans) >= 2
            assert all(code in (4, 5, 6) for _, code in rejected)
            assert all(any(len(g) > 1 for g in pl) for pl in plans)
            if boxes:
                assert _fuses_boxed(prog, plans[0])


def test_run_launch_count():
    """sp_run_launch_count: one launch per live launch on one rank; on several ranks the
    launches that receive ghost planes split into interior + boundary (C4 fused, 2 ranks:
    only the first launch receives the step-start exchange)."""
    import json
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    from synth.scale_les import c4
    prog = c4(nx=64, ny=32, nz=32)
    plan = json.load(open(os.path.join(ROOT, "configs", "c4_plan.json")))["groups"]
    p = Program(prog)
    p.set_plan(plan)
    assert p.launch_count("fused") == len(plan)
    assert p.launch_count("unfused") == len(prog["kernels"])
    comms = Comm.loopback(2)
    q = Program(prog, comm=comms[0], nz_global=64, z_offset=0, zhalo=4)
    q.set_plan(plan)
    recv = [i for i in range(len(plan)) if q.exchange_plan("fused", i)]
    assert recv
    assert q.launch_count("fused") == len(plan) + len(recv)


def test_lazy_fission_search_model_objective():
    """sp_plan_search_ex (NEXT #1) with the model objective: deterministic,
    legal, never worse than its exact contiguous-segmentation DP seed, which is never
    worse than the unfused plan; on C4 (no kernel needs fission) no kernel is split, on
    C3 the search fissions K0's two independent outputs (P and Q, Fig.-3 style) and fuses
    one of them with its consumer."""
    from synth.scale_les import c4
    for name, prog in (("C4", c4(nx=256, ny=32, nz=64)), ("C3", P.c3())):
        p = Program(prog)
        plan, rep = p.plan_search_ex(generations=15, population=12, seed=2)
        assert (plan, rep) == p.plan_search_ex(generations=15, population=12, seed=2)
        p.set_plan(plan)
        refs = [r for g in plan for r in g]
        assert len(refs) == len(set(refs)) == sum(len(k["stmts"]) for k in prog["kernels"])
        assert rep["cost_us"] <= rep["dp_cost_us"] + 1e-9 <= rep["unfused_cost_us"] + 1e-9
        assert rep["generations_run"] == 15 and rep["groups_evaluated"] > len(prog["kernels"])
        if name == "C4":
            assert rep["fissioned_kernels"] == 0
        else:
            assert rep["fissioned_kernels"] == 1
            k0 = [g for g in plan if any(r.startswith("K0:") for r in g)]
            assert len(k0) == 2 and any(len(g) > 1 for g in k0)


def test_bench_refuses_gpu_count_mismatch():
    """bench.py never reports an N-GPU run that is not one: --gpus != WORLD_SIZE
    under torchrun, or --gpus N > visible devices without it, exits non-zero before any work."""
    import subprocess
    import sys
    bench = os.path.join(ROOT, "bench.py")
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, bench, "--gpus", "4"], capture_output=True, text=True, env=env,
                       timeout=120)
    assert r.returncode != 0 and "WORLD_SIZE=2" in r.stderr
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env["CUDA_VISIBLE_DEVICES"] = ""
    r = subprocess.run([sys.executable, bench, "--gpus", "2"], capture_output=True, text=True, env=env,
                       timeout=300)
    assert r.returncode != 0 and "CUDA device" in r.stderr


def test_exchange_schedule_includes_boxed_stage_previous_value():
    """Reading R2' on several ranks: a boxed statement evaluated on a plane beyond the slab
    (lead 1 here: K2's T2 is read one plane above by K3) loads T2's previous value outside
    its box there, so the schedule receives T2's ghost plane above (and nothing below),
    besides A's step-start planes; without loop bounds T2 is never exchanged (it is
    computed on chip everywhere)."""
    from paper_conf_hpdc_wahibm15_b200 import Comm
    prog = P.resize(P.chain3(), 20, 12, 12)
    comms = Comm.loopback(2)
    q = Program(prog, comm=comms[0], nz_global=24, z_offset=0, zhalo=2)
    q.set_plan(prog["plans"]["fused"])
    assert [x for x in q.exchange_plan("fused", 0) if x[0] == "T2"] == []
    prog["kernels"][1]["box"] = [2, 17, 1, 10, 8, 20]
    q = Program(prog, comm=comms[0], nz_global=24, z_offset=0, zhalo=2)
    q.set_plan(prog["plans"]["fused"])
    assert ("T2", 0, 1) in q.exchange_plan("fused", 0)


def test_live_out_stores_writer_before_boxed_rewrite():
    """Reading R2' / R6: when a later group rewrites X only inside a box, the earlier
    writer of X must store it (the boxed statement loads the old value outside its box) —
    the bug the round-2 legal-plan fuzz exposed.  Here T (a TEMP) is written by K1 and
    rewritten in a box by K2 in the next group, then read by K3: group 0 stores T."""
    T = P.tap
    prog = {"name": "boxlive", "dtype": "f64", "grid": {"nx": 8, "ny": 6, "nz": 4, "ghost": [1, 1, 1]},
            "arrays": [{"name": n, "role": r} for n, r in (("A", "in"), ("T", "temp"), ("O", "out"))],
            "kernels": [P.kernel("K1", P.stmt("T", [{"c": 2.0, "a": T("A", (0, 0, 0))}])),
                        dict(P.kernel("K2", P.stmt("T", [{"c": 3.0, "a": T("A", (1, 0, 0))}])),
                             box=[1, 4, 0, 6, 0, 4]),
                        P.kernel("K3", P.stmt("O", [{"c": 1.0, "a": T("T", (0, 0, 0))}]))]}
    p = Program(prog)
    p.set_plan([["K1"], ["K2", "K3"]])
    assert p.report("fused", 0)["n_stores"] == 1
    p.set_plan([["K1"], ["K2"], ["K3"]])
    assert [r["n_stores"] for r in p.reports("fused")] == [1, 1, 1]


@pytest.mark.parametrize("name", ["C2", "C3", "C5"])
def test_frame_mode_codegen_and_pins(name):
    """Option / pin "frame": region-vector evaluation replaces the point-wise halo strips
    (no per-thread halo tables in the source), units are 16-byte x-vectors, the tile
    height is free of the thread count, and the kernels compile for sm_100a."""
    prog = P.CONFIGS[name]()
    plan = prog["plans"]["fission_fused" if name == "C3" else "fused"]
    p = Program(prog, options={"frame": 1})
    p.set_plan(plan)
    src = p.source("fused")
    assert "fi_" in src and "_f[i]" not in src
    vw = 16 // (4 if prog["dtype"] == "f32" else 8)
    assert all(r["block_x"] == vw and r["block_y"] == 1 for r in p.reports("fused"))
    p.compile("fused")
    assert all(0 < r["regs_per_thread"] <= 255 for r in p.reports("fused"))
    # a per-launch pin with a tile height no block geometry could give
    p.tune("fused", 0, dict(tile_x=32, tile_y=5, threads=64, zchunk=8, frame=1))
    r = p.report("fused", 0)
    assert (r["tile_x"], r["tile_y"], r["threads"]) == (32, 5, 64)
    # and the pin can switch it off again for that launch only
    p.tune("fused", 0, dict(frame=0))
    assert "_f[i]" in p.source("fused")


def test_frame2_queues_and_fallback():
    """frame=2: one unit grid per launch with register queues for own-position taps
    (input queues "zg_", stage queues "rq" beside the shared-memory rings); a shape whose
    queues cannot fit in 255 registers falls back to frame mode 1 instead of failing."""
    prog = P.c3(n=64)
    p = Program(prog, options={"frame": 2})
    p.set_plan(prog["plans"]["fission_fused"])
    g0 = p.source("fused").split("sf_fused_1")[0]
    assert "zg_I" in g0 and "rq0[" in g0 and "fi_" in g0
    p.tune("fused", 0, dict(tile_x=64, tile_y=16, threads=32, zchunk=8, frame=2))
    r = p.report("fused", 0)
    g0 = p.source("fused").split("sf_fused_1")[0]
    assert (r["tile_x"], r["tile_y"], r["threads"]) == (64, 16, 32)
    assert "fi_" in g0 and "zg_I" not in g0      # frame mode 1 at that shape
    p.compile("fused")


def test_producer_wait_variants_codegen():
    """The TMA producer waits for a free ring slot with nanosleep back-off by default
    (option psleep, ns), spins with psleep=0, or uses a try_wait suspend hint (phint);
    the role test is warp-uniform (shuffle broadcast of the warp index)."""
    prog = P.c2(n=64)
    for opts, want in (({}, "sf_mbar_wait_backoff(&empty"), ({"psleep": 0}, "sf_mbar_wait(&empty"),
                       ({"phint": 5000}, "sf_mbar_wait_hint(&empty")):
        p = Program(prog, options=opts)
        p.set_plan(prog["plans"]["fused"])
        src = p.source("fused")
        assert want in src, opts
        assert "__shfl_sync(0xffffffffu, tid >> 5, 0) >= NT / 32" in src
    p.compile("fused")


def test_ring_and_barrier_options_codegen():
    """pow2ring rounds every ring depth up to a power of two (more shared memory, a mask
    slot); pbar signals "slot free" through named barriers (compute warps bar.arrive, the
    whole producer warp bar.sync, ids 2..2+NE-1) instead of the empty mbarriers."""
    prog = P.c3(n=64)
    p = Program(prog)
    p.set_plan(prog["plans"]["fission_fused"])
    base = [r["smem_bytes"] for r in p.reports("fused")]
    q = Program(prog, options={"pow2ring": 1})
    q.set_plan(prog["plans"]["fission_fused"])
    assert all(b2 >= b1 for b1, b2 in zip(base, [r["smem_bytes"] for r in q.reports("fused")]))
    src = q.source("fused")
    import re
    depths = {int(d) for d in re.findall(r"% (\d+)u\) \*", src)}
    assert depths and all(d & (d - 1) == 0 for d in depths), depths
    b = Program(prog, options={"pbar": 1})
    b.set_plan(prog["plans"]["fission_fused"])
    src = b.source("fused")
    assert "sf_bar_arrive(2 + ((k - KF)" in src and "sf_bar_sync(2 + ((s - KF)" in src
    assert "sf_mbar_arrive(&empty" not in src
    b.compile("fused")


def test_launch_dag_with_temp_renaming():
    """sp_plan_dag: with TEMP renaming (default) C4's diag groups become roots and only the
    real data flow orders the groups; without it every group hangs on its predecessors'
    TEMP reuse (WAR/WAW); streams follow the latest dependency; slabs of a decomposed
    grid and the unfused mode never rename."""
    from synth.scale_les import c4
    import json
    prog = c4(nx=64, ny=32, nz=16)
    plan = json.load(open(os.path.join(ROOT, "configs", "c4_plan.json")))["groups"]
    p = Program(prog)
    p.set_plan(plan)
    dag = p.dag()
    assert [d for d, _ in dag] == [[], [0], [], [0, 2], [], [2, 3, 4], [], [4, 6], [], [6, 8]]
    assert {s for _, s in dag} == {0, 1}
    for i, (d, s) in enumerate(dag):
        if d:
            assert s == dag[d[-1]][1]
    q = Program(prog, options={"rename": 0, "streams": 1})
    q.set_plan(plan)
    dq = q.dag()
    assert all(i == 0 or (i - 1) in d for i, (d, _) in enumerate(dq))  # a chain
    assert {s for _, s in dq} == {0}
    slab = Program(prog, nz_global=32, z_offset=0, zhalo=4)
    slab.set_plan(plan)
    assert all(i == 0 or (i - 1) in d for i, (d, _) in enumerate(slab.dag()))
    assert all(s == 0 for _, s in p.dag("unfused"))
