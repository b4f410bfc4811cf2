"""Print the per-shape table of a column-suite detail JSON."""
import json
import sys

d = json.load(open(sys.argv[1]))
print(d["value"], "min best/auto", d["min_shape_best_over_auto"], d["config"]["thresholds"])
f = lambda v: ("%8.1f" % v) if v is not None else "    None"
for r in d["shapes"]:
    print(f"{r['op']:8s} n=2^{r['n'].bit_length()-1:2d} ch={r['chosen']:6s} auto={f(r['auto'])} top={f(r['top'])} "
          f"mid={f(r['middle'])} flat={f(r['flat'])} b/a={r['best_over_auto']:.3f} GB/s={r['GBps']}")
