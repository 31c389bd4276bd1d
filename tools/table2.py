"""Per-group occupancy table (the paper's Table 2 analogue; NEXT #4), host only.

python tools/table2.py C4 gpurun_out/occ_C4.csv [--plan fused] [--md out.md]

The CSV is an ncu --csv capture of tools/prof_step.py <workload> --steps 1 --warmup 1
(-k regex:sf_fused) with the metrics of METRICS below; each launch appears twice, the
second occurrence is used.  Theoretical occupancy is what the launch configuration
allows (ncu sm__maximum_warps_per_active_cycle_pct); achieved is sm__warps_active.
The algorithmic GB/s use the byte model of sp_plan_report.
"""
import argparse
import csv
import io
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "sm__warps_active.avg.pct_of_peak_sustained_active",
           "sm__maximum_warps_per_active_cycle_pct", "launch__occupancy_limit_shared_mem",
           "launch__occupancy_limit_registers", "launch__registers_per_thread",
           "launch__block_size", "launch__grid_size", "launch__waves_per_multiprocessor"]


def load(path):
    text = open(path).read()
    text = text[text.index('"ID"'):]
    per = {}
    for r in csv.DictReader(io.StringIO(text)):
        key = (r["ID"], r["Kernel Name"])
        per.setdefault(key, {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    out = {}
    for (_, name), m in sorted(per.items(), key=lambda kv: int(kv[0][0])):
        out[name] = m  # the later occurrence wins
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("csv")
    ap.add_argument("--plan", default="fused")
    ap.add_argument("--md")
    a = ap.parse_args()
    import bench
    from paper_conf_hpdc_wahibm15_b200 import Program
    prog = bench.load_workload(a.workload)
    p = Program(prog)
    p.set_plan(bench.plan_of(prog, a.plan))
    bench.apply_tuning(p, prog, a.plan)
    reps = p.reports("fused")
    groups = bench.plan_of(prog, a.plan)
    m = load(a.csv)
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    lines = [f"# {a.workload} ({a.plan}): per-group occupancy and bandwidth (ncu, B200)", "",
             "| launch | stmts | tile x zc, threads | regs | CTAs/SM (smem, regs) | theor. occ. | "
             "achieved occ. | waves | time us | alg GB/s | DRAM GB/s |", "|" + "---|" * 11]
    tot_t = 0.0
    for i, r in enumerate(reps):
        k = f"sf_fused_{i}"
        if k not in m:
            continue
        x = m[k]
        t = x["gpu__time_duration.sum"] / 1e3  # ns -> us
        tot_t += t
        dram = (x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"])
        alg = r["bytes_alg"] * pts
        lines.append(
            f"| {k} | {len(groups[i])} | {r['tile_x']}x{r['tile_y']}x{r['zchunk']}, {r['threads']} | "
            f"{int(x['launch__registers_per_thread'])} | {int(x['launch__occupancy_limit_shared_mem'])}, "
            f"{int(x['launch__occupancy_limit_registers'])} | {x['sm__maximum_warps_per_active_cycle_pct']:.1f} % | "
            f"{x['sm__warps_active.avg.pct_of_peak_sustained_active']:.1f} % | "
            f"{x['launch__waves_per_multiprocessor']:.2f} | {t:.1f} | {alg / t / 1e3:.0f} | {dram / t / 1e3:.0f} |")
    lines += ["", f"Sum of launch times {tot_t:.1f} us (ncu, serialised, --clock-control none)."]
    text = "\n".join(lines) + "\n"
    print(text)
    if a.md:
        open(a.md, "w").write(text)


if __name__ == "__main__":
    main()
