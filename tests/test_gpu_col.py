"""GPU parity for the column (axis-0) reduce / scan, the left-hand side of
rule G4: every version through the C ABI against
the oracle's column loops.  Bar as for rows: int32 and f32
min/max bit-exact; f32 sums within 1e-5 * (sum_i |f(x_ij)| + |d|); F32_EXACT
inputs bit-exact for every version."""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "flat", "auto"]
SHAPES = [(1, 1), (7, 5), (33, 37), (300, 128), (1000, 64), (64, 4100), (3, 10003), (4096, 3), (5000, 1),
          (257, 96),
          # narrow V_FLAT (m | 32, n*m % 32 == 0: virtual 32-wide rows, stride-m warp scans)
          (4096, 4), (8192, 1), (2080, 16), (1056, 2), (96, 8), (1024, 64), (4096, 32), (1000, 8), (4095, 32)]


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


def dev(x, misalign=False):
    if not misalign:
        return x.cuda()
    buf = torch.empty(x.numel() + 1, dtype=x.dtype, device="cuda")
    xd = buf[1:].view(x.shape)
    xd.copy_(x)
    return xd


def check(orc, x, got, scan, op, f="id", d=None):
    xn = x.cpu().numpy()
    g = got.cpu().numpy()
    if xn.dtype == np.int32 or op in ("min", "max"):
        want = orc.colscan(xn, op, f, d) if scan else orc.colred(xn, op, f, d)
        np.testing.assert_array_equal(g, want.astype(g.dtype))
        return
    want, ab = orc.colscan(xn, op, f, d, with_absum=True)
    if not scan:
        want, ab = want[-1], ab[-1]
    bound = 1e-5 * (ab + (0.0 if d is None else abs(float(d))))
    err = np.abs(g.astype(np.float64) - want)
    assert (err <= bound).all(), f"max err {err.max():.3g} (bound there {bound.flat[err.argmax()]:.3g})"


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
def test_col_shapes_i32_f32(ifl, orc, version, scan):
    fn = ifl.colscan if scan else ifl.colred
    for (n, m) in SHAPES:
        for mis in (False, True):
            xi = gen.matrix("I32_FULL", 31, n, m)
            check(orc, xi, fn(dev(xi, mis), "sum", version=version), scan, "sum")
            xf = gen.matrix("F32_SIGNED", 32, n, m)
            check(orc, xf, fn(dev(xf, mis), "sum", version=version), scan, "sum")


@pytest.mark.parametrize("version", VERS)
def test_col_ops_maps_neutral(ifl, orc, version):
    n, m = 129, 68
    xi = gen.matrix("I32_FULL", 33, n, m)
    for op in ("sum", "prod", "min", "max", "and", "or", "xor"):
        for f in ("id", "sq", "abs"):
            for scan in (False, True):
                fn = ifl.colscan if scan else ifl.colred
                check(orc, xi, fn(xi.cuda(), op, f, version=version), scan, op, f)
    xf = gen.matrix("F32_SIGNED", 34, n, m)
    for op in ("sum", "min", "max"):
        for scan in (False, True):
            fn = ifl.colscan if scan else ifl.colred
            check(orc, xf, fn(xf.cuda(), op, "sq", ne=0.25, version=version), scan, op, "sq", 0.25)
            check(orc, xi, fn(xi.cuda(), op, ne=7, version=version), scan, op, "id", 7)


@pytest.mark.parametrize("scan", [False, True])
def test_col_exact_all_versions_bitwise(ifl, orc, scan):
    # F32_EXACT: every partial sum is an integer < 2^24, so every order is exact
    for (n, m) in [(4099, 36), (20000, 4), (50, 20000), (65536, 2)]:
        x = gen.matrix("F32_EXACT", 35, n, m)
        want = (orc.colscan if scan else orc.colred)(x.numpy())
        for v in VERS:
            got = (ifl.colscan if scan else ifl.colred)(x.cuda(), version=v).cpu().numpy()
            np.testing.assert_array_equal(got, want.astype(np.float32))


def test_col_g4_identity_on_gpu(ifl):
    # G4: column reduce = segred of the transpose, on the device
    x = gen.matrix("I32_FULL", 36, 700, 300).cuda()
    for v in VERS:
        assert torch.equal(ifl.colred(x, "xor", version=v), ifl.segred(x.t().contiguous(), "xor"))
        assert torch.equal(ifl.colscan(x, "sum", version=v), ifl.segscan(x.t().contiguous(), "sum").t())


def test_col_empty_inplace_and_large(ifl, orc):
    e = torch.empty(0, 5, dtype=torch.int32, device="cuda")
    assert ifl.colred(e, "min").cpu().tolist() == [2**31 - 1] * 5  # reduce of [] = d
    assert ifl.colscan(e).shape == (0, 5)
    assert ifl.colred(torch.empty(5, 0, device="cuda")).numel() == 0
    x = gen.matrix("I32_FULL", 37, 513, 260).cuda()
    want = ifl.colscan(x, version="middle")
    for v in VERS:  # in place (out == in)
        y = x.clone()
        ifl.colscan(y, out=y, version=v)
        assert torch.equal(y, want)
    # bench-sized shapes (2^26 elements), sampled columns against the oracle
    for (n, m) in [(1 << 13, 1 << 13), (1 << 22, 16), (16, 1 << 22), (1 << 26, 1), (1 << 20, 64)]:
        xf = gen.matrix("F32_SIGNED", 38, n, m)
        cols = np.unique(np.r_[0, m // 3, m - 1])
        sub = np.ascontiguousarray(xf.numpy()[:, cols])
        want, ab = orc.colscan(sub, with_absum=True)
        xd = xf.cuda()
        for v in ("middle", "flat", "auto"):
            got = ifl.colred(xd, version=v).cpu().numpy()[cols]
            assert (np.abs(got - want[-1]) <= 1e-5 * ab[-1]).all(), (n, m, v)
            gs = ifl.colscan(xd, version=v)[:, cols].cpu().numpy()
            assert (np.abs(gs - want) <= 1e-5 * ab).all(), (n, m, v, "scan")
