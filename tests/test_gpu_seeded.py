"""GPU parity of ifl_segscan_seeded (per-row d, the carry-in of a column
block) against oracle.segscan_seeded, every version and every kernel path
(TOP m in {1,2,4} / {8,16,32} / tiled, MIDDLE, FLAT short and long rows,
misaligned inputs), plus the split-row identity the multi-GPU inner split
relies on."""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "cluster", "flat", "auto"]
SHAPES = [(7, 1), (9, 2), (13, 4), (45, 8), (70, 16), (33, 32), (50, 33), (300, 100), (3, 7000), (2, 30001),
          (1, 200000), (4000, 37)]


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


def _check(orc, x, seed, got, op):
    xn, sn, g = x.cpu().numpy(), seed.cpu().numpy(), got.cpu().numpy()
    if x.dtype == torch.int32:
        np.testing.assert_array_equal(g, orc.segscan_seeded(xn, sn, op))
        return
    want, ab = orc.segscan_seeded(xn, sn, op, with_absum=True)
    if op in ("min", "max"):
        np.testing.assert_array_equal(g, want.astype(np.float32))
    else:
        err = np.abs(g.astype(np.float64) - want)
        assert (err <= 1e-5 * ab).all(), float(err.max())


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("dt,op", [("i32", "sum"), ("i32", "max"), ("i32", "xor"), ("f32", "sum"), ("f32", "min")])
def test_seeded_parity(ifl, orc, version, dt, op):
    for k, (n, m) in enumerate(SHAPES):
        x = gen.matrix("I32_FULL" if dt == "i32" else "F32_SIGNED", 40 + k, n, m)
        seed = gen.matrix("I32_FULL" if dt == "i32" else "F32_SIGNED", 90 + k, 1, n).view(n).contiguous()
        got = ifl.segscan(x.cuda(), op, seed=seed.cuda(), version=version)
        _check(orc, x, seed, got, op)


@pytest.mark.parametrize("version", ["top", "middle", "flat"])
def test_seeded_misaligned(ifl, orc, version):
    n, m = 37, 301
    x = gen.matrix("I32_FULL", 3, n, m)
    buf = torch.empty(n * m + 1, dtype=torch.int32, device="cuda")
    xd = buf[1:].view(n, m)
    xd.copy_(x)
    seed = gen.matrix("I32_FULL", 4, 1, n).view(n).contiguous()
    _check(orc, x, seed, ifl.segscan(xd, "sum", seed=seed.cuda(), version=version), "sum")


@pytest.mark.parametrize("version", ["top", "middle", "flat"])
def test_split_row_identity(ifl, version):
    # scan of columns [k, m) seeded with column k-1 of the full scan == tail
    # of the full scan (int32: bit-exact)
    n, m = 6, 50000
    x = gen.matrix("I32_FULL", 8, n, m).cuda()
    full = ifl.segscan(x, "sum", version="flat")
    for k in (1, 4097, 33333):
        tail = ifl.segscan(x[:, k:].contiguous(), "sum", seed=full[:, k - 1].contiguous(), version=version)
        assert torch.equal(tail, full[:, k:])


def test_seeded_rejects_bad_seed(ifl):
    x = torch.zeros(4, 8, dtype=torch.int32, device="cuda")
    with pytest.raises(ValueError):
        ifl.segscan(x, "sum", seed=torch.zeros(3, dtype=torch.int32, device="cuda"))
    with pytest.raises(ValueError):
        ifl.segscan(x, "sum", seed=torch.zeros(4, dtype=torch.float32, device="cuda"))
