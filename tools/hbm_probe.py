"""HBM context probe (not part of the product): torch copy and torch sum
bandwidth on 1 GiB fp32, CUDA events, best of 10.  Tells what read-only
streaming can reach on this B200 next to the driver's copy peak."""
import json

import torch

x = torch.rand(1 << 28, device="cuda")
y = torch.empty_like(x)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def best(fn, nbytes, reps=10):
    fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return nbytes / (min(ts) / 1e3) / 1e9


r = {"copy_GBps": best(lambda: y.copy_(x), 2 * x.numel() * 4),
     "sum_GBps": best(lambda: x.sum(), x.numel() * 4),
     "rowsum_1024_GBps": best(lambda: x.view(-1, 1024).sum(1), x.numel() * 4),
     "cumsum_GBps": best(lambda: torch.cumsum(x, 0, out=y), 2 * x.numel() * 4, reps=3)}
print(json.dumps(r))
