"""Merge a tools/tune_workload.py result for the 'unfused' plan into configs/<w>_plan.json.

python tools/merge_unfused.py C2 tune.json
C4's frozen-plan file keeps them as unfused_configs; the other workloads' files carry
them under plans["unfused"] (bench.load_workload reads both forms).
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
w, src = sys.argv[1], sys.argv[2]
t = json.load(open(src))["plans"]["unfused"]
path = os.path.join(ROOT, "configs", f"{w.lower()}_plan.json")
pj = json.load(open(path)) if os.path.exists(path) else {"workload": w, "plans": {}}
if w == "C4":
    pj["unfused_configs"], pj["unfused_group_us"] = t["configs"], t["group_us"]
else:
    pj.setdefault("plans", {})["unfused"] = {"configs": t["configs"], "group_us": t["group_us"]}
pj["unfused_tuner"] = "tools/tune_workload.py <w> unfused --quick (isolated launches, clean L2), B200"
json.dump(pj, open(path, "w"), indent=1)
print("merged", len(t["configs"]), "unfused configs ->", path, "sum", round(sum(t["group_us"]), 1), "us")
