"""V_FLAT irregular segred + segscan at ~2^26 elements (targets for ncu launch
lists and captures; not part of the product).  argv: mean [reps]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

mean = float(sys.argv[1]) if len(sys.argv) > 1 else 1024.0
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
off = gen.irregular_offsets(5, int((1 << 26) // mean), mean)
offd = torch.from_numpy(off).cuda()
total = int(off[-1])
x = gen.generate("F32_UNIT", 2, total, "cuda")
for _ in range(reps):
    ifl.segred_irr(x, offd, version="flat")
    ifl.segscan_irr(x, offd, version="flat")
torch.cuda.synchronize()
