import sys; sys.path.insert(0,'.')
import numpy as np, torch
import ifl_inputs as gen
import paper_conf_ppopp_henriksenteo19_b200 as ifl
ifl.reset_thresholds()
off = gen.irregular_offsets(11, 20000, 40.0)
offd = torch.from_numpy(off).cuda()
x = gen.generate("F32_EXACT", 92, int(off[-1]))
for scan in (False, True):
    for v in ["top","middle","flat","auto"]:
        got = (ifl.segscan_irr if scan else ifl.segred_irr)(x.cuda(), offd, version=v).cpu()
        torch.cuda.synchronize(); print(scan, v, 'ok', flush=True)
xr = gen.matrix("I32_FULL", 93, 300, 77).cuda()
offr = (torch.arange(301, dtype=torch.int64) * 77).cuda()
for v in ["top","middle","flat","auto"]:
    a=ifl.segred_irr(xr.view(-1), offr, "xor", version=v); torch.cuda.synchronize(); print('irr red', v, flush=True)
    c=ifl.segred(xr, "xor"); torch.cuda.synchronize(); print('reg red', flush=True)
    print(torch.equal(a, c))
    b=ifl.segscan_irr(xr.view(-1), offr, version=v); torch.cuda.synchronize(); print('irr scan', v, flush=True)
    c=ifl.segscan(xr); torch.cuda.synchronize(); print('reg scan', flush=True)
    print(torch.equal(b, c.view(-1)))
