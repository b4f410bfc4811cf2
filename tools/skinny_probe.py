"""redomap2 V_FLAT on the skinny end of the Fig 2 family (n = p = 2^a,
m = 2^(k-2a)): time (CUDA graph), GB/s of the algorithmic bytes, and a
float64 torch check (not the parity test) -- both B layouts."""
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402


def gtime(fn, R=3):
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(R):
            fn()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(3):
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / R)
    return statistics.median(ts)


for dt, k, amax in (("bf16", 30, 7), ("f32", 25, 6), ("f32", 28, 6)):
    tdt = torch.bfloat16 if dt == "bf16" else torch.float32
    s = 2 if dt == "bf16" else 4
    for a in range(0, amax + 1):
        n = p = 1 << a
        m = 1 << (k - 2 * a)
        A = gen.generate("BF16_SIGNED", 6, n * m, device="cuda").view(n, m).to(tdt)
        Bt = gen.generate("BF16_SIGNED", 7, p * m, device="cuda").view(p, m).to(tdt)
        B = Bt.t().contiguous()
        C = torch.empty(n, p, device="cuda")
        ws = ifl.workspace(ifl.workspace_bytes("redomap2", n, m, p, dt), "cuda", "mm")
        ref = (A.double() @ Bt.double().t()).float()
        byts = s * (n * m + m * p) + 4 * n * p
        r = {"dt": dt, "k": k, "n": n, "m": m}
        for name, BB, km in (("kmaj", Bt, True), ("rowmaj", B, False)):
            t = gtime(lambda: ifl.redomap2(A, BB, b_kmajor=km, out=C, ws=ws, version="flat"))
            err = (C - ref).abs().max().item() / max(1e-30, (A.double().abs() @ Bt.double().abs().t()).max().item())
            r[name + "_us"] = round(t * 1e3, 1)
            r[name + "_GBps"] = round(byts / t / 1e6)
            r[name + "_relerr"] = float(f"{err:.2e}")
        print(json.dumps(r), flush=True)
        del A, Bt, B, C, ref
        torch.cuda.empty_cache()
