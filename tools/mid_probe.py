"""Time V_MIDDLE segred on the configs[1] sweep shapes with few rows (the
cluster-per-row path), CUDA-graph timed, two alternating inputs."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench_suites as bs  # noqa: E402
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

N = 1 << 26
x = gen.generate("F32_UNIT", 2, N, device="cuda")
out = torch.empty(N, device="cuda")
res = {"lib": os.environ.get("IFL_LIB_PATH", "default").split("/")[-1]}
for n in [int(a) for a in (sys.argv[1:] or [2, 4, 8, 16, 32])]:
    m = N // n
    res[n] = round(bs.gtime(lambda: ifl.segred(x.view(n, m), out=out[:n], version="middle")) * 1e3, 1)
print(json.dumps(res))
