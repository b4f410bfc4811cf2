"""Run one (op, version, n, m) configuration a few times -- a small target
for `ncu -k regex:... --set full` (not part of the product)."""
import argparse
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--op", default="segred")
ap.add_argument("--version", default="flat")
ap.add_argument("--n", type=int, default=1)
ap.add_argument("--m", type=int, default=1 << 26)
ap.add_argument("--p", type=int, default=1, help="redomap2: columns of C; tridag: coefficient rows R")
ap.add_argument("--dt", default="bf16", help="redomap2 input dtype")
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
if a.op == "redomap2":
    tdt = torch.bfloat16 if a.dt == "bf16" else torch.float32
    A = gen.generate("BF16_SIGNED", 6, a.n * a.m, device="cuda").view(a.n, a.m).to(tdt)
    Bt = gen.generate("BF16_SIGNED", 7, a.p * a.m, device="cuda").view(a.p, a.m).to(tdt)
    C = torch.empty(a.n, a.p, device="cuda")
    ws = ifl.workspace(ifl.workspace_bytes("redomap2", a.n, a.m, a.p, a.dt), "cuda", "mm")
    x = None

    def fn(_x, version):
        return ifl.redomap2(A, Bt, out=C, ws=ws, version=version)
elif a.op == "tridag":
    ta, tb, tc, ty = (t.cuda() for t in gen.tridag_system(7, a.n, a.m, a.p))
    tx = torch.empty_like(ty)
    ws = ifl.workspace(ifl.workspace_bytes("tridag", a.n, a.m, a.p), "cuda", "tri")
    x = None

    def fn(_x, version):
        return ifl.tridag(ta, tb, tc, ty, out=tx, ws=ws, version=version)
elif a.op == "lvc":  # --n numS --m numX --p numY, numT = 64
    xc, yc, xs, ys = gen.lvc_problem(17, a.n, a.m, a.p, "cuda")
    x = None

    def fn(_x, version):
        return ifl.lvc(xs, ys, xc, yc, 64, version=version)
elif a.op in ("colred", "colscan"):
    x = gen.generate("F32_UNIT", 2, a.n * a.m, device="cuda").view(a.n, a.m)
    fn = ifl.colred if a.op == "colred" else ifl.colscan
elif a.op in ("segred_irr", "segscan_irr"):  # --m = mean segment length, ~2^26 elements
    off = gen.irregular_offsets(5, max(1, (1 << 26) // a.m), float(a.m))
    offd = torch.from_numpy(off).cuda()
    xi = gen.generate("F32_UNIT", 2, int(off[-1]), device="cuda")
    mx = ifl.irr_inspect(offd, int(off[-1]))
    x = None
    g = ifl.segred_irr if a.op == "segred_irr" else ifl.segscan_irr

    def fn(_x, version):
        return g(xi, offd, version=version, max_len=mx)
else:
    x = gen.generate("F32_UNIT", 2, a.n * a.m, device="cuda").view(a.n, a.m)
    fn = ifl.segred if a.op == "segred" else ifl.segscan
for _ in range(a.reps):
    fn(x, version=a.version)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
fn(x, version=a.version)
e1.record()
torch.cuda.synchronize()
print(f"{a.op} {a.version} n={a.n} m={a.m}: {e0.elapsed_time(e1)*1e3:.1f} us")
