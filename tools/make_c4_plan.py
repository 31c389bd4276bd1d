"""Freeze the greedy fission/fusion plan of C4 to configs/c4_plan.json (host-side, no GPU)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402
from synth.scale_les import c4  # noqa: E402

prog = c4()
p = Program(prog)
plan = p.plan_greedy()
p.set_plan(plan)
fused = sum(r["bytes_alg"] for r in p.reports("fused")) / p.elem
unfused = sum(r["bytes_alg"] for r in p.reports("unfused")) / p.elem
out = {"workload": "C4", "planner": "greedy (sp_plan_greedy)", "groups": plan,
       "passes": {"fused": fused, "unfused": unfused}}
json.dump(out, open(os.path.join(ROOT, "configs", "c4_plan.json"), "w"), indent=1)
print(f"{len(plan)} groups, passes {unfused:.0f} -> {fused:.0f}")
