"""Flat-engine timing probe (not the product bench): V_FLAT segred and
segscan on the configs[1] sweep shapes that use it, CUDA-graph timed with two
alternating resident inputs (> L2).  IFL_LIB_PATH selects an experiment
build of the library."""
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

N = 1 << 26
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
    return statistics.median(ts)


tag = os.environ.get("IFL_LIB_PATH", "default").split("/")[-1]
res = {"lib": tag}
for n in [int(a) for a in (sys.argv[1:] or [1, 64, 4096, 8192, 262144])]:
    m = N // n
    tr = gtime(lambda c: ifl.segred(xs[c].view(n, m), out=out[:n], ws=ws, version="flat"))
    ts = gtime(lambda c: ifl.segscan(xs[c].view(n, m), out=out.view(n, m), ws=ws, version="flat"))
    tm = gtime(lambda c: ifl.segscan(xs[c].view(n, m), out=out.view(n, m), ws=ws, version="middle")) if n >= 4096 else None
    res[n] = {"red_us": round(tr, 1), "scan_us": round(ts, 1), "scan_mid_us": None if tm is None else round(tm, 1),
              "red_GBps": round(4 * (N + n) / tr / 1e3), "scan_GBps": round(8 * N / ts / 1e3)}
print(json.dumps(res), flush=True)
