"""Per-window step times over a long back-to-back run, with nvidia-smi samples (dev tool).

python tools/step_series.py C4 --steps 400 --window 20
"""
import argparse
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("workload")
ap.add_argument("--steps", type=int, default=400)
ap.add_argument("--window", type=int, default=20)
ap.add_argument("--mode", default="fused")
a = ap.parse_args()
prog = bench.load_workload(a.workload)
dev = torch.device("cuda:0")
p = Program(prog)
p.set_plan(bench.plan_of(prog))
bench.apply_tuning(p, prog)
p.allocate(dev, fill=0.0)
bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
for _ in range(10):
    p.run(a.mode)
torch.cuda.synchronize()
log = "/tmp/step_series_smi.csv"
proc = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=timestamp,clocks.sm,clocks.mem,power.draw,"
                         "temperature.gpu,temperature.memory,clocks_event_reasons.active",
                         "--format=csv,noheader", "-lms", "20", "-f", log])
time.sleep(0.3)
ev = [torch.cuda.Event(enable_timing=True) for _ in range(a.steps // a.window + 1)]
ev[0].record()
for w in range(1, len(ev)):
    for _ in range(a.window):
        p.run(a.mode)
    ev[w].record()
torch.cuda.synchronize()
time.sleep(0.1)
proc.terminate()
print("window ms/step:", " ".join(f"{ev[w - 1].elapsed_time(ev[w]) / a.window:.3f}"
                                  for w in range(1, len(ev))))
print("total", ev[0].elapsed_time(ev[-1]) / (a.window * (len(ev) - 1)))
time.sleep(0.2)
for ln in open(log):
    print(ln.strip())
