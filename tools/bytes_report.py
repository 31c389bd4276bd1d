"""Per-launch DRAM bytes (ncu) against the byte model, fused and unfused (host only).

python tools/bytes_report.py C4 gpurun_out/bytes_C4.csv [--plan fused] [--json out.json]

The CSV is an ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,
dram__bytes_write.sum -k regex:sf_ capture of tools/prof_step.py --unfused --steps 1
--warmup 1 (each launch twice; the second occurrence is used).  The model's
algorithmic bytes are elem x (|ExtIn| + |LiveOut|) per point,
executed bytes add halo re-reads and z warm-up.  Per-launch DRAM writes are split
unevenly between neighbouring launches (L2 write-back happens late), so the step
totals are the comparison that counts; per launch it is indicative.
"""
import argparse
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402


def read_ncu(path):
    lines = open(path).read().splitlines()
    start = [i for i, l in enumerate(lines) if l.startswith('"ID"')][0]
    rows = list(csv.reader(lines[start:]))
    hdr = rows[0]
    ki, mi, vi, ui, ii = (hdr.index(h) for h in ("Kernel Name", "Metric Name", "Metric Value",
                                                  "Metric Unit", "ID"))
    by_id = collections.OrderedDict()
    for r in rows[1:]:
        d = by_id.setdefault(r[ii], {"kernel": r[ki]})
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6,
                 "usecond": 1e-6, "nsecond": 1e-9, "msecond": 1e-3}.get(unit, 1)
        d[r[mi]] = v * scale
    last = {}
    for d in by_id.values():  # keep the last occurrence of each kernel
        last[d["kernel"]] = d
    return last


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("csv")
    ap.add_argument("--plan", default="fused")
    ap.add_argument("--json", default=None)
    a = ap.parse_args()
    prog = bench.load_workload(a.workload)
    p = Program(prog)
    p.set_plan(bench.plan_of(prog, a.plan))
    bench.apply_tuning(p, prog, a.plan)
    g = prog["grid"]
    pts = g["nx"] * g["ny"] * g["nz"]
    meas = read_ncu(a.csv)
    out = {"workload": a.workload, "plan": a.plan, "source": os.path.basename(a.csv), "modes": {}}
    for mode in ("unfused", "fused"):
        rows = []
        for i, r in enumerate(p.reports(mode)):
            name = f"sf_{mode}_{i}"
            if r["grid_ctas"] == 0 or name not in meas:
                continue
            m = meas[name]
            dram = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
            rows.append({"launch": name, "alg_bytes": r["bytes_alg"] * pts,
                         "exec_bytes": r["bytes_exec"] * pts, "dram_bytes": dram,
                         "time_us": m.get("gpu__time_duration.sum", 0) * 1e6})
        tot = {k: sum(x[k] for x in rows) for k in ("alg_bytes", "exec_bytes", "dram_bytes", "time_us")}
        out["modes"][mode] = {"launches": rows, "total": tot}
    u, f = out["modes"]["unfused"]["total"], out["modes"]["fused"]["total"]
    out["reduction"] = {"model_alg": 1 - f["alg_bytes"] / u["alg_bytes"],
                        "dram_measured": 1 - f["dram_bytes"] / u["dram_bytes"],
                        "time_serialised": 1 - f["time_us"] / u["time_us"]}
    for mode in ("unfused", "fused"):
        t = out["modes"][mode]["total"]
        print(f"{a.workload} {mode:8s} launches {len(out['modes'][mode]['launches']):3d}  alg "
              f"{t['alg_bytes']/1e9:7.3f} GB  exec {t['exec_bytes']/1e9:7.3f} GB  DRAM "
              f"{t['dram_bytes']/1e9:7.3f} GB ({t['dram_bytes']/t['alg_bytes']:.2f}x alg)  "
              f"{t['time_us']:8.1f} us (ncu, serialised)")
    r = out["reduction"]
    print(f"{a.workload} traffic reduction: model {r['model_alg']*100:.1f} %, measured DRAM "
          f"{r['dram_measured']*100:.1f} %, time {r['time_serialised']*100:.1f} %")
    if a.json:
        json.dump(out, open(a.json, "w"), indent=1)


if __name__ == "__main__":
    main()
