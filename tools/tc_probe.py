"""Dense bf16 squares through the tcgen05 kernel (redomap2 V_TOP): TFLOP/s,
CUDA-graph timed; cuBLAS beside it as context."""
import json
import statistics
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402


def gtime(fn, R=5):
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
    for _ in range(5):
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / R)
    return statistics.median(ts)


for q in [int(a) for a in sys.argv[1:]] or [2048, 4096, 8192]:
    A = gen.generate("BF16_SIGNED", 6, q * q, device="cuda").view(q, q).to(torch.bfloat16)
    Bt = gen.generate("BF16_SIGNED", 7, q * q, device="cuda").view(q, q).to(torch.bfloat16)
    C = torch.empty(q, q, device="cuda")
    ws = ifl.workspace(ifl.workspace_bytes("redomap2", q, q, q, "bf16"), "cuda", "mm")
    t = gtime(lambda: ifl.redomap2(A, Bt, out=C, ws=ws, version="top"))
    tc = gtime(lambda: torch.matmul(A, Bt.t()))
    B = Bt.t().contiguous()  # yss [m][p]: the MN-major operand path (b_kmajor = 0)
    trm = gtime(lambda: ifl.redomap2(A, B, b_kmajor=False, out=C, ws=ws, version="top"))
    print(json.dumps({"q": q, "us": round(t * 1e3, 1), "TFLOPs": round(2 * q**3 / t / 1e9, 1),
                      "rowmajor_B_us": round(trm * 1e3, 1), "rowmajor_over_kmajor": round(trm / t, 3),
                      "cublas_TFLOPs": round(2 * q**3 / tc / 1e9, 1)}), flush=True)
