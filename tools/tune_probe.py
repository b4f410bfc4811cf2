"""Print the tuner's cost table (ms per version) for a site on the bench's
training sweeps (n*m = 2^25 and 2^27) and the chosen thresholds."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

site = sys.argv[1] if len(sys.argv) > 1 else "segred.b4"
train = [(1 << k, 1 << (lg - k)) for lg in (25, 27) for k in range(lg + 1)]
need = ifl.lib().ifl_tune_scratch_bytes(site.encode(), np.asarray(train, np.int64).ctypes.data, len(train))
scratch = torch.empty(need, dtype=torch.uint8, device="cuda")
scratch.view(-1)[: (need // 4) * 4].view(torch.float32).copy_(gen.generate("F32_UNIT", 4, need // 4, "cuda"))
a, b, tbl = ifl.tune(site, train, reps=3, cost=1, scratch=scratch)
print(site, "t_top", a, "t_intra", b)
for (n, m), row in zip(train, tbl):
    c = ifl.select(site, n, m)
    print(f"n*m=2^{(n*m).bit_length()-1} n=2^{n.bit_length()-1:2d} top={row[0]*1e3:10.1f} mid={row[1]*1e3:9.1f} "
          f"flat={row[2]*1e3:8.1f} chosen={c.version}")
