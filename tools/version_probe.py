"""Per-version timing probe (not the product bench): segred / segscan, every
forced version, on sweep shapes n = 2^k (n*m = 2^26), CUDA-graph timed with two
alternating resident inputs (> L2).  IFL_LIB_PATH selects an experiment build.
    python tools/version_probe.py k1 k2 ... [--ops segred,segscan] [--versions top,middle,flat]"""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("ks", type=int, nargs="*", default=[18, 20, 21, 22, 23, 24])
ap.add_argument("--ops", default="segred,segscan")
ap.add_argument("--versions", default="top,middle,flat")
ap.add_argument("--log2n", type=int, default=26)
a = ap.parse_args()
N = 1 << a.log2n
xs = [gen.generate("F32_UNIT", 2, N, device="cuda"), gen.generate("F32_UNIT", 3, N, device="cuda")]
out = torch.empty(N, device="cuda")
ws = ifl.workspace(ifl.workspace_bytes("segscan", 1, N), "cuda")


def gtime(fn, R=4):
    fn(0)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for r in range(R):
            fn(r % 2)
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(5):
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / R * 1e3)
    return round(statistics.median(ts), 1)


res = {"lib": os.environ.get("IFL_LIB_PATH", "libifl.so").split("/")[-1]}
for k in a.ks:
    n, m = 1 << k, N >> k
    row = {}
    for op in a.ops.split(","):
        for v in a.versions.split(","):
            if op == "segred":
                f = lambda c: ifl.segred(xs[c].view(n, m), out=out[:n], ws=ws, version=v)  # noqa: E731
            else:
                f = lambda c: ifl.segscan(xs[c].view(n, m), out=out.view(n, m), ws=ws, version=v)  # noqa: E731
            row[f"{op[3:]}_{v[0]}"] = gtime(f)
    res[k] = row
print(json.dumps(res), flush=True)
