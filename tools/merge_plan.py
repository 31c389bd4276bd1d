"""Derive a plan variant by merging adjacent groups of a frozen plan (dev tool).

python tools/merge_plan.py configs/c4_plan.json 0+1 4+5 --out /tmp/p.json
Configurations of untouched groups are carried over; merged groups get None
(tile chooser) until tools/step_tune.py --groups tunes them.
"""
import argparse
import json

ap = argparse.ArgumentParser()
ap.add_argument("plan")
ap.add_argument("merges", nargs="*")
ap.add_argument("--out", required=True)
a = ap.parse_args()
pj = json.load(open(a.plan))
groups, cfgs = pj["groups"], pj.get("configs") or [None] * len(pj["groups"])
spans = sorted(tuple(int(v) for v in m.split("+")) for m in a.merges)
out_g, out_c, i = [], [], 0
while i < len(groups):
    span = next((s for s in spans if s[0] == i), None)
    if span:
        assert list(span) == list(range(span[0], span[-1] + 1)), "merge adjacent groups only"
        out_g.append([m for j in span for m in groups[j]])
        out_c.append(None)
        i = span[-1] + 1
    else:
        out_g.append(groups[i])
        out_c.append(cfgs[i])
        i += 1
pj.update(groups=out_g, configs=out_c, planner=pj.get("planner", "") + f" + merges {a.merges}")
pj.pop("group_ms", None)
json.dump(pj, open(a.out, "w"), indent=1)
print(len(out_g), "groups ->", a.out, [i for i, c in enumerate(out_c) if c is None])
