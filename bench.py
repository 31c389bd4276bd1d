"""Benchmark of the fused stencil-DAG executor (driver contract).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C4] [--impl ours|reference]

One step = one pass of the whole hot path over the workload: every group of the
fusion plan (run_fused: on one rank along the group dependency DAG on two streams, TEMPs
renamed per writer group; on N > 1 ranks in plan order), plus on N > 1 ranks the z-slab
halo exchanges.  Metric (BASELINE.json): grid-point updates/s (interior points x
original kernels / s, reading R21) and HBM GB/s against the roofline, fused vs
unfused.  N > 1: one process per GPU (torchrun), z-slab decomposition, weak
scaling (per-GPU grid fixed).  Inputs: seeded synthetic fields (synth/), 2.1 GB
per GPU for C4 (larger than the 126 MB L2, so no flush between steps).

--impl reference times the CPU oracle (oracle/, the plain serial program) on a
bounded sample of the same workload, as the reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "grid-point updates/s and HBM GB/s (% of roofline), fused vs unfused, 1/2/4/8 B200"
UNIT = "grid-point updates/s"


def load_workload(name):
    """Program dict of a workload.  Frozen plans and tuned per-launch configurations
    (measured on B200 with tools/ab_plans.py / tools/step_tune.py) come from
    configs/<workload>_plan.json: C4's plan is the measured-greedy planner output;
    the other workloads keep their hand plans (synth/programs.py) and only carry
    configurations, keyed by plan name."""
    from synth import programs as P
    if name == "C4":
        from synth.scale_les import c4
        prog = c4()
        # SF_C4_PLAN: candidate plan file for A/B runs (dev tools); default the frozen plan
        plan_path = os.environ.get("SF_C4_PLAN") or os.path.join(ROOT, "configs", "c4_plan.json")
        if os.path.exists(plan_path):
            pj = json.load(open(plan_path))
            prog["plans"]["fused"] = pj["groups"]
            prog["plan_configs"] = {"fused": pj.get("configs"), "unfused": pj.get("unfused_configs")}
        return prog
    prog = P.CONFIGS[name]()
    path = os.path.join(ROOT, "configs", f"{name.lower()}_plan.json")
    if os.path.exists(path):
        pj = json.load(open(path))
        prog["plan_configs"] = {k: v.get("configs") for k, v in pj["plans"].items()}
        for k, v in pj["plans"].items():  # searched plans (e.g. "measured") carry their groups
            if v.get("groups"):
                prog["plans"][k] = v["groups"]
    return prog


def tuned_configs(prog, plan="fused"):
    return (prog.get("plan_configs") or {}).get(plan)


def apply_tuning(p, prog, plan="fused"):
    cfgs = tuned_configs(prog, plan)
    if cfgs:
        for i, c in enumerate(cfgs):
            if c:
                p.tune("fused", i, c)
    # the unfused baseline's per-kernel configurations, when tuned
    for i, c in enumerate(tuned_configs(prog, "unfused") or []):
        if c:
            p.tune("unfused", i, c)


def plan_of(prog, name="fused"):
    if name in prog["plans"]:
        return prog["plans"][name]
    from paper_conf_hpdc_wahibm15_b200 import Program
    return Program(prog).plan_greedy()


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index):
        self.idx = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.idx), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.time()  # nvidia-smi takes a moment to start: wait for its first sample
            while not self.lines and time.time() - t0 < 3.0 and self.proc.poll() is None:
                time.sleep(0.02)
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self, min_samples=3):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        t0 = time.time()  # a short timed region still gets a few samples around it
        while len(self.lines) < min_samples and time.time() - t0 < 1.0:
            time.sleep(0.02)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[2:]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(sm)}


def fill_inputs(p, prog, device, z_offset, zhalo):
    from synth.fields import field_torch
    hz = p.ghost[2]
    extra = (zhalo - hz, zhalo - hz)
    for aid, a in enumerate(prog["arrays"]):
        v = field_torch(4, aid, p.n, p.ghost, prog["dtype"], device, z_offset=z_offset,
                        nz_alloc_extra=extra)
        p.padded_view(p.tensors[a["name"]], hz=zhalo).copy_(v)


def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_hpdc_wahibm15_b200 import Comm, Program

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("SF_BENCH_SHARE_GPU") == "1" and world > 1:
        # functional test of the N > 1 path on ONE GPU (tests/test_gpu_nccl.py): every rank
        # on cuda:0, NCCL told the ranks sit on different hosts (socket transport over
        # loopback); the numbers of such a run measure nothing and are labelled so
        local = 0
        os.environ.update({"NCCL_HOSTID": f"stencilfuse-rank{rank}", "NCCL_SOCKET_IFNAME": "lo",
                           "NCCL_IB_DISABLE": "1", "NCCL_P2P_DISABLE": "1", "NCCL_SHM_DISABLE": "1",
                           "NCCL_NVLS_ENABLE": "0"})
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local if world > 1 else 0)
    torch.cuda.set_device(dev)
    prog = load_workload(args.workload)
    plan = plan_of(prog, args.plan)
    nz = prog["grid"]["nz"]
    # deep halo needed by the plan's accumulated z-reach (probe on the local grid)
    probe = Program(prog)
    probe.set_plan(plan)
    apply_tuning(probe, prog, args.plan)
    reach = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused") for r in probe.reports(m)] +
                [prog["grid"]["ghost"][2]])
    zhalo = reach if world > 1 else prog["grid"]["ghost"][2]
    del probe
    comm = Comm(rank, world) if world > 1 else None
    xpush = bool(args.xpush and world > 1)
    if xpush and os.environ.get("SF_BENCH_SHARE_GPU") == "1":
        # peer-push kernels spin on flags the neighbour's kernels set; ranks sharing one
        # GPU have no co-residency guarantee (Xid 109 recorded on this driver)
        raise SystemExit("--xpush needs one GPU per rank (not with SF_BENCH_SHARE_GPU=1)")
    p = Program(prog, comm=comm, nz_global=nz * world, z_offset=rank * nz, zhalo=zhalo,
                options={"xpush": 1} if xpush else None)
    p.set_plan(plan)
    apply_tuning(p, prog, args.plan)
    p.allocate(dev, fill=0.0)
    fill_inputs(p, prog, dev, rank * nz, zhalo)
    if xpush:
        p.connect_peers(rank, world)
        # every rank's modules are loaded before any kernel can wait on a neighbour
        # (a neighbour still compiling would otherwise look like a dead rank)
        p.load("fused")
        p.load("unfused")
        torch.cuda.synchronize(dev)
        dist.barrier()
    stream = torch.cuda.current_stream(dev)
    n_pts = prog["grid"]["nx"] * prog["grid"]["ny"] * nz  # per GPU
    n_kernels = len(prog["kernels"])
    reps_f = p.reports("fused")
    reps_u = p.reports("unfused")
    live_f = [i for i, r in enumerate(reps_f) if r["grid_ctas"] > 0]

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---------------------------------------------------------- fused, timed
    for _ in range(args.warmup):
        p.run_fused(stream)
    barrier()
    sampler = ClockSampler(dev.index)
    sampler.start()
    time.sleep(0.25)
    per_launch = [0.0] * len(reps_f)
    # headline: K steps back to back (launches adjacent on the stream, so programmatic
    # dependent launch overlaps each group's prologue with the previous group's tail)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    t0 = time.perf_counter()
    s.record(stream)
    for k in range(args.steps):
        p.run_fused(stream)
    e.record(stream)
    barrier()
    wall = time.perf_counter() - t0
    step_ms = s.elapsed_time(e) / args.steps
    clocks = sampler.stop()
    step_ms = max_over_ranks(step_ms)
    # sustained: >= 1 s of back-to-back steps (at least 200), one CUDA event per step
    # boundary on the launching stream; median / mean per step beside the K-step headline
    sus_n = max(200, int(1.0 / max(step_ms * 1e-3, 1e-6)) + 1)
    sus_ev = [torch.cuda.Event(enable_timing=True) for _ in range(sus_n + 1)]
    sus_sampler = ClockSampler(dev.index)
    sus_sampler.start()
    time.sleep(0.25)
    barrier()
    sus_ev[0].record(stream)
    for k in range(sus_n):
        p.run_fused(stream)
        sus_ev[k + 1].record(stream)
    barrier()
    sus_clocks = sus_sampler.stop()
    per_step = [sus_ev[k].elapsed_time(sus_ev[k + 1]) for k in range(sus_n)]
    sustained = {"steps": sus_n, "ms_per_step_median": max_over_ranks(statistics.median(per_step)),
                 "ms_per_step_mean": max_over_ranks(sus_ev[0].elapsed_time(sus_ev[-1]) / sus_n),
                 "timed_s": sus_ev[0].elapsed_time(sus_ev[-1]) * 1e-3, "clocks": sus_clocks}
    # the same step captured once as a CUDA graph and replayed K times (SURVEY.md §8(d)
    # timing protocol; S7): launch overhead off the host, same kernels
    graph_ms = None
    try:
        g = torch.cuda.CUDAGraph()
        gs = torch.cuda.Stream(device=dev)
        gs.wait_stream(stream)
        with torch.cuda.stream(gs):
            with torch.cuda.graph(g, stream=gs):
                p.run_fused(gs)
        barrier()
        g.replay()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        barrier()
        s.record(stream)
        for k in range(args.steps):
            g.replay()
        e.record(stream)
        barrier()
        graph_ms = max_over_ranks(s.elapsed_time(e) / args.steps)
        del g
    except Exception as ex:  # reported, never silently replacing the headline
        graph_ms = f"capture failed: {ex}"
    # per-launch durations (dominant kernel of the roofline): a second timed pass of
    # the same launches with CUDA events between them on the launching stream
    prof_steps = max(3, min(args.steps, 50))
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(len(live_f) + 1)]
           for _ in range(prof_steps)]
    barrier()
    for k in range(prof_steps):
        for j, i in enumerate(live_f):
            evs[k][j].record(stream)
            p.run_launch("fused", i, stream)
        evs[k][-1].record(stream)
    barrier()
    for j, i in enumerate(live_f):
        per_launch[i] = sum(evs[k][j].elapsed_time(evs[k][j + 1])
                            for k in range(prof_steps)) / prof_steps

    # ---------------------------------------------------------- unfused, same K
    for _ in range(args.warmup):
        p.run_unfused(stream)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    s.record(stream)
    for _ in range(args.steps):
        p.run_unfused(stream)
    e.record(stream)
    barrier()
    unf_ms = max_over_ranks(s.elapsed_time(e) / args.steps)

    # ---------------------------------------------------------- e2e through the public API
    in_names = [a["name"] for a in prog["arrays"] if a["role"] in ("in", "inout")]
    out_names = [a["name"] for a in prog["arrays"] if a["role"] in ("out", "inout")]
    host_in = {n: torch.empty_like(p.tensors[n], device="cpu").pin_memory() for n in in_names}
    host_out = {n: torch.empty_like(p.tensors[n], device="cpu").pin_memory() for n in out_names}
    for n in in_names:
        host_in[n].copy_(p.tensors[n])
    e2e_steps = max(2, min(args.steps, 10))
    # Pipelined through the public API: step k's inputs go host->device on one copy
    # stream and step k-1's outputs device->host on another while step k-1 computes;
    # inputs and outputs are double-buffered and rebound (stencil_program_bind) per step.
    dev_in = [{n: p.tensors[n] for n in in_names},
              {n: torch.empty_like(p.tensors[n]) for n in in_names}]
    dev_out = [{n: p.tensors[n] for n in out_names},
               {n: dev_in[1][n] if n in in_names else torch.empty_like(p.tensors[n])
                for n in out_names}]
    for n in out_names:  # ghost cells of the second output buffer (never written by kernels)
        if n not in in_names:
            dev_out[1][n].copy_(p.tensors[n])
    h2d_s, d2h_s = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
    in_ready = [torch.cuda.Event() for _ in range(e2e_steps)]
    done = [torch.cuda.Event() for _ in range(e2e_steps)]
    out_read = [torch.cuda.Event() for _ in range(e2e_steps)]
    barrier()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record(stream)
    h2d_s.wait_event(s)
    d2h_s.wait_event(s)
    for k in range(e2e_steps):
        b = k % 2
        with torch.cuda.stream(h2d_s):
            if k >= 2:
                h2d_s.wait_event(done[k - 2])       # buffer b no longer read by step k-2
            for n in in_names:
                dev_in[b][n].copy_(host_in[n], non_blocking=True)
            in_ready[k].record(h2d_s)
        stream.wait_event(in_ready[k])
        if k >= 2:
            stream.wait_event(out_read[k - 2])       # outputs of step k-2 copied out
        for n in in_names:
            p.bind(n, dev_in[b][n])
        for n in out_names:
            p.bind(n, dev_out[b][n])
        p.run_fused(stream)
        done[k].record(stream)
        with torch.cuda.stream(d2h_s):
            d2h_s.wait_event(done[k])
            for n in out_names:
                host_out[n].copy_(dev_out[b][n], non_blocking=True)
            out_read[k].record(d2h_s)
    stream.wait_event(out_read[e2e_steps - 1])
    e.record(stream)
    barrier()
    e2e_ms = max_over_ranks(s.elapsed_time(e) / e2e_steps)
    for n in in_names:
        p.bind(n, dev_in[0][n])
    for n in out_names:
        p.bind(n, dev_out[0][n])
    h2d = sum(host_in[n].numel() * host_in[n].element_size() for n in in_names)
    d2h = sum(host_out[n].numel() * host_out[n].element_size() for n in out_names)

    # ---------------------------------------------------------- report (rank 0)
    if rank == 0:
        pk = peaks()
        peak = pk["hbm_gbs"] if pk else 6650.0
        peak_src = "MEASURED_PEAKS.json hbm_gbs (measured copy)" if pk else "fallback 6.65 TB/s"
        updates = n_pts * world * n_kernels
        value = updates / (step_ms * 1e-3)
        # dominant kernel: largest share of the step
        dom = max(live_f, key=lambda i: per_launch[i])
        r = reps_f[dom]
        achieved = r["bytes_alg"] * n_pts / (per_launch[dom] * 1e-3) / 1e9
        traffic = None
        tp = os.path.join(ROOT, "profiles", f"ncu_traffic_{args.workload}.json")
        if os.path.exists(tp):
            traffic = json.load(open(tp)).get(f"sf_fused_{dom}")
        alg_step = sum(x["bytes_alg"] for x in reps_f) * n_pts
        alg_step_u = sum(x["bytes_alg"] for x in reps_u) * n_pts
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": prog["dtype"], "data": "synthetic: seeded splitmix64 uniform[-1,1) fields",
            "config": {"workload": args.workload, "grid_per_gpu": [prog["grid"]["nx"], prog["grid"]["ny"], nz],
                       "kernels": n_kernels, "arrays": len(prog["arrays"]),
                       "plan": args.plan, "fused_groups": len(live_f),
                       # the fused step's launch DAG (TEMP renaming + streams, one rank)
                       "launch_streams": (1 + max(st for _, st in p.dag("fused"))) if world == 1 else 1,
                       "parallelism": f"z-slab x{world}",
                       "halo_exchange": ("peer-push (TEMP) + NCCL (step-start)" if xpush else
                                         "NCCL send/recv") if world > 1 else "none",
                       "l2": "no flush: per-GPU working set > 126 MB L2"},
            **({"functional_test": "SF_BENCH_SHARE_GPU=1: all ranks share one GPU; not a measurement"}
               if os.environ.get("SF_BENCH_SHARE_GPU") == "1" else {}),
            "hbm_gbs_alg": alg_step / (step_ms * 1e-3) / 1e9,
            # the launches one at a time in plan order (the per-launch pass) against the step,
            # which runs them along the group DAG: what the concurrency recovers
            "launch_dag": {"serial_launch_sum_ms": sum(per_launch[i] for i in live_f),
                           "step_ms": step_ms},
            "roofline_step": {"achieved": alg_step / (step_ms * 1e-3) / 1e9, "peak": peak,
                              "unit": "GB/s", "frac": alg_step / (step_ms * 1e-3) / 1e9 / peak,
                              "frac_of_8tbs_nominal": alg_step / (step_ms * 1e-3) / 8e12},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "kernel": f"sf_fused_{dom}",
                         "share_of_step": per_launch[dom] / step_ms, "peak_source": peak_src},
            "fused_vs_unfused": {"unfused_ms_per_step": unf_ms,
                                 "unfused_value": updates / (unf_ms * 1e-3),
                                 "speedup": unf_ms / step_ms,
                                 "bytes_alg_per_step": {"fused": alg_step, "unfused": alg_step_u},
                                 "predicted_traffic_reduction": 1 - alg_step / alg_step_u},
            "e2e": {"value": updates / (e2e_ms * 1e-3), "unit": UNIT, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": e2e_ms},
            "sustained": dict(sustained, value=updates / (sustained["ms_per_step_median"] * 1e-3),
                              frac_of_peak=alg_step / (sustained["ms_per_step_median"] * 1e-3) / 1e9 / peak,
                              note="median of per-step CUDA events over >= 1 s of back-to-back steps"),
            "graph_replay": {"ms_per_step": graph_ms, "note": "one fused step captured as a CUDA "
                             "graph, replayed K times (same kernels; not the headline)"},
            # this library's kernels in the timed region (sp_run_launch_count: on N > 1 a
            # launch that receives ghost planes is an interior + one boundary launch)
            "gpu_launches": args.steps * p.launch_count("fused"),
            "clocks": clocks,
            "wall_s_timed": wall,
        }
        if world == 1 and not args.no_cpu:
            line["cpu_baseline"] = cpu_baseline(args, budget_s=15.0)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def oracle_step_time(prog, nz_s, seed=4, parallel=False):
    from oracle import OracleProgram, dense_arrays
    from synth.programs import resize
    g = prog["grid"]
    sub = resize(prog, g["nx"], g["ny"], nz_s)
    arrs = dense_arrays(sub, seed)
    o = OracleProgram(sub, parallel=parallel)
    t0 = time.perf_counter()
    o.run(arrs)
    return time.perf_counter() - t0, sub


def cpu_baseline(args, budget_s=15.0, steps=1):
    """The oracle (single thread, as it stands) on a z-subslab of the workload."""
    prog = load_workload(args.workload)
    g = prog["grid"]
    t1, _ = oracle_step_time(prog, 1)
    per_plane = max(t1, 1e-4)
    nz_s = int(max(1, min(g["nz"], budget_s / per_plane / max(steps, 1))))
    steps = max(steps, int(budget_s / (per_plane * nz_s)))  # whole slab fits: repeat it
    ts = []
    for _ in range(steps):
        t, sub = oracle_step_time(prog, nz_s)
        ts.append(t)
    t = sum(ts) / len(ts)
    upd = g["nx"] * g["ny"] * nz_s * len(prog["kernels"])
    out = {"value": upd / t, "unit": UNIT, "cores": 1, "kind": "oracle",
           "sample": f"{args.workload} program on a {g['nx']}x{g['ny']}x{nz_s} z-(sub)slab, mean of {steps} "
                     f"step(s), serial C oracle (-O2 -ffp-contract=off), {t:.2f} s per step"}
    # context only: the OpenMP build of the same loop nest on every
    # host core, on the whole per-GPU slab (identical results, tests/test_oracle_pins.py)
    try:
        cores = os.cpu_count() or 1
        tp, _ = oracle_step_time(prog, g["nz"], parallel=True)
        out["parallel"] = {"value": g["nx"] * g["ny"] * g["nz"] * len(prog["kernels"]) / tp,
                           "unit": UNIT, "cores": cores,
                           "kind": "oracle loop nest, OpenMP over z (-fopenmp), one step"}
    except Exception as e:  # reported, not fatal
        out["parallel"] = f"unavailable: {e}"
    return out


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    prog = load_workload(args.workload)
    g = prog["grid"]
    t1, _ = oracle_step_time(prog, 1)
    budget = 150.0 / max(args.steps + args.warmup, 1)
    nz_s = int(max(1, min(g["nz"], budget / max(t1, 1e-4))))
    for _ in range(args.warmup):
        oracle_step_time(prog, nz_s)
    ts = [oracle_step_time(prog, nz_s)[0] for _ in range(args.steps)]
    t = sum(ts) / len(ts)
    upd = g["nx"] * g["ny"] * nz_s * len(prog["kernels"])
    v = upd / t
    sample = (f"{args.workload} program on a {g['nx']}x{g['ny']}x{nz_s} z-subslab per step, "
              f"serial C oracle, 1 thread")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": prog["dtype"],
        "data": "synthetic", "config": {"workload": args.workload,
                                        "grid_per_gpu": [g["nx"], g["ny"], g["nz"]]},
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def _free_port():
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    return port


def ensure_world(args):
    """One process per GPU.  Under torchrun (WORLD_SIZE set) the world must equal --gpus;
    without it, --gpus N > 1 re-executes this script under torch.distributed.run with N
    ranks on this node (the driver's own launch line) and exits with its status, so a
    multi-GPU request never silently benchmarks one GPU."""
    env = os.environ.get("WORLD_SIZE")
    if env is not None:
        if int(env) != args.gpus:
            sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={env}: refusing to report a "
                     f"{env}-rank run as {args.gpus} GPUs")
        return
    if args.gpus <= 1:
        return
    if args.impl == "ours" and os.environ.get("SF_BENCH_SHARE_GPU") != "1":
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            sys.exit(f"bench.py: --gpus {args.gpus} requested but only {have} CUDA device(s) visible")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1",
           f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--workload", default="C4", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--plan", default="fused", help="named plan of the workload (e.g. C3 fission_fused)")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--xpush", action="store_true",
                    help="N > 1: peer-push halo exchange of TEMP epochs (CUDA IPC over NVLink, "
                         "in-kernel progress protocol) instead of NCCL send/recv for them")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus < 1:
        sys.exit("bench.py: --gpus must be >= 1")
    ensure_world(args)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
