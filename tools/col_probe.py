"""Run colred/colscan V_FLAT once on a few sweep shapes (for an ncu launch list)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

x = gen.generate("F32_UNIT", 2, 1 << 26, "cuda")
out = torch.empty_like(x)
for (n, m) in [(1 << 26, 1), (1 << 20, 64), (1 << 16, 1024)]:
    for fn in (ifl.colred, ifl.colscan):
        o = out.view(n, m) if fn is ifl.colscan else out[:m]
        fn(x.view(n, m), out=o, version="flat")
torch.cuda.synchronize()
