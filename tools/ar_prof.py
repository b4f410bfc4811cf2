"""Phase timers of the AR flat-scan engine (variant build with -DIFL_AR_PROF)."""
import ctypes
import sys

import torch

sys.path.insert(0, ".")
import ifl_inputs as gen  # noqa: E402
import paper_conf_ppopp_henriksenteo19_b200 as ifl  # noqa: E402

N = 1 << 26
x = gen.generate("F32_UNIT", 2, N, device="cuda")
out = torch.empty(N, device="cuda")
ws = ifl.workspace(ifl.workspace_bytes("segscan", 1, N), "cuda")
L = ifl.lib()
buf = (ctypes.c_ulonglong * 16)()
names = ["scan_cons_wait_full", "scan_cons_lookback", "scan_total(x2)", "scan_prod_wait_agg", "scan_prod_wait_empty",
         "agg_prod_flowctl", "agg_prod_wait_empty", "agg_cons_wait_full", "agg_total(x2)", "scan_bulk_wait_read",
         "n_agg", "n_scan"]
for n in [int(a) for a in sys.argv[1:]] or [1, 4096, 65536]:
    m = N // n
    for _ in range(3):
        ifl.segscan(x.view(n, m), out=out.view(n, m), ws=ws, version="flat")
    torch.cuda.synchronize()
    L.ifl_debug_prof(buf)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    R = 5
    e0.record()
    for _ in range(R):
        ifl.segscan(x.view(n, m), out=out.view(n, m), ws=ws, version="flat")
    e1.record()
    torch.cuda.synchronize()
    L.ifl_debug_prof(buf)
    na, ns = buf[10] / R, buf[11] / R
    us = e0.elapsed_time(e1) / R * 1e3
    print(f"n={n} {us:.1f} us/call  agg CTAs {na:.0f} scan CTAs {ns:.0f}")
    for i in range(10):
        per = buf[i] / R / (na if "agg" in names[i] else ns) / 1.9e3
        if "total" in names[i]:
            per /= 2
        print(f"   {names[i]:24s} {per:8.1f} us per CTA")
