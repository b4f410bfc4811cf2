"""Time ifl_lvc V_OUTER on the P:402 datasets (graph-timed), for A/B of
kernel variants (IFL_LVC_IT=16 forces 16 items per lane)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench_suites as bs  # noqa: E402
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

out = {"IT_env": os.environ.get("IFL_LVC_IT")}
for ds, (S, T, X, Y) in gen.LVC_DATASETS.items():
    xc, yc, xs, ys = gen.lvc_problem(17, S, X, Y, "cuda")
    out[ds] = round(bs.gtime(lambda: ifl.lvc(xs, ys, xc, yc, T, version="outer"), R=2) * 1e3, 1)
print(json.dumps(out))
