"""redomap2 timing probe (not the product bench): every version on the
configs[2] family and dense squares, CUDA-graph timed; cuBLAS (torch.matmul)
beside it as context only."""
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


rows = []
dts = sys.argv[1:] or ["bf16", "f32"]
for dt in dts:
    tdt = torch.bfloat16 if dt == "bf16" else torch.float32
    s = 2 if dt == "bf16" else 4
    shapes = [(1 << a, 1 << (30 - 2 * a), 1 << a) for a in range(0, 16)] if dt == "bf16" else \
             [(1 << a, 1 << (28 - 2 * a), 1 << a) for a in range(0, 15)]
    shapes += [(q, q, q) for q in (1024, 2048, 4096, 8192)]
    for (n, m, p) in shapes:
        A = gen.generate("BF16_SIGNED", 6, n * m, device="cuda").view(n, m).to(tdt)
        Bt = gen.generate("BF16_SIGNED", 7, p * m, device="cuda").view(p, m).to(tdt)
        C = torch.empty(n, p, device="cuda")
        ws = ifl.workspace(ifl.workspace_bytes("redomap2", n, m, p, dt), "cuda", "mm")
        r = {"dt": dt, "n": n, "m": m, "p": p}
        for v in ("top", "middle", "flat", "auto"):
            if v != "auto" and v != "top" and n * p > (1 << 22):
                continue  # warp/CTA per output with > 4M outputs: minutes; skipped
            if v == "middle" and m >= (1 << 24):
                continue
            if v == "top" and dt == "f32" and n * p < 64 and m >= (1 << 22):
                continue  # SIMT TOP on a degenerate grid: seconds
            t = gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws, version=v))
            r[v + "_us"] = t * 1e3
        r["cublas_us"] = gtime(lambda: torch.matmul(A, Bt.t(), out=None)) * 1e3 if dt == "bf16" else None
        flops = 2.0 * n * m * p
        byts = s * (n * m + m * p) + 4 * n * p
        r.setdefault("top_us", float("nan"))
        r["auto_TFLOPs"] = flops / (r["auto_us"] * 1e-6) / 1e12
        r["auto_GBps"] = byts / (r["auto_us"] * 1e-6) / 1e9
        r["chosen"] = ifl.redomap2(A, Bt, out=C, ws=ws, return_choice=True)[1].version
        rows.append(r)
        print(json.dumps(r), flush=True)
        del A, Bt, C
