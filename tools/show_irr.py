"""Print the per-shape table of an irregular-suite detail JSON."""
import json
import sys

d = json.load(open(sys.argv[1]))
print(d["value"], "min best/auto", d["min_shape_best_over_auto"], d["config"]["thresholds"])
for r in d["shapes"]:
    print(f"{r['op']:8s} mean={r['mean']:6d} n={r['n']:9d} max={r['max_len']:8d} ch={r['chosen']:6s} "
          f"auto={r['auto']:8.1f} top={r['top']:9.1f} mid={r['middle']:9.1f} flat={r['flat']:8.1f} "
          f"b/a={r['best_over_auto']:.3f} GB/s={r['GBps']}")
