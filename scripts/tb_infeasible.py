"""Per order: stencils on which an OC was infeasible for every setting (the paper's
"crash"), from a label dataset written by scripts/label_dataset.py."""
import collections
import json
import math
import sys

for path in sys.argv[1:]:
    lab = [json.loads(l) for l in open(path)]
    lab = [r for r in lab if r.get("kind") != "setting"]
    inf = collections.Counter()
    tot = collections.Counter()
    for r in lab:
        order = r["features"]["order"]
        tot[order] += 1
        for name, t in r["oc_times_ms"].items():
            if t is None or (isinstance(t, float) and math.isinf(t)):
                inf[(order, name)] += 1
    print(path, "stencils per order:", dict(sorted(tot.items())))
    for (o, n), c in sorted(inf.items()):
        print(f"  order {o}: {n} infeasible on {c}")
