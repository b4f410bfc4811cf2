import sys, torch, numpy as np
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import ifl_inputs as gen, paper_conf_ppopp_henriksenteo19_b200 as ifl
lg, mean = int(sys.argv[1]), float(sys.argv[2])
n = max(1, (1 << lg) // int(mean))
off = gen.irregular_offsets(224, n, mean)
offd = torch.from_numpy(off).cuda(); total = int(off[-1])
print("n", n, "total", total, "max", np.diff(off).max(), "empty frac", (np.diff(off) == 0).mean(), flush=True)
x = gen.generate("F32_UNIT", 5, total, "cuda")
for kind in ("segred", "segscan"):
    for v in ("top", "middle", "flat"):
        fn = ifl.segscan_irr if kind == "segscan" else ifl.segred_irr
        fn(x, offd, version=v); torch.cuda.synchronize(); print(kind, v, "ok", flush=True)
