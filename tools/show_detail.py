"""Print the per-shape table of a bench detail JSON (bench.py --detail)."""
import json
import sys

d = json.load(open(sys.argv[1]))
ln = d["line"]
print(sys.argv[1], ln["value"], "min best/auto", ln.get("min_shape_best_over_auto"))
for r in d["table"]:
    print(f"{r['op']:8s} n=2^{r['n'].bit_length()-1:2d} ch={r['chosen']:6s} auto={r['auto_us']:8.1f} "
          f"top={r['top_us']:9.1f} mid={r['middle_us']:9.1f} flat={r['flat_us']:9.1f} "
          f"b/a={r['best_over_auto']:.3f} GB/s={r['auto_GBps']:.0f}")
