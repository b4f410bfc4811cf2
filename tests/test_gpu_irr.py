"""GPU parity for irregular segments: every
version of ifl_segred_irr / ifl_segscan_irr through the C ABI against the
oracle's per-segment loops.  Bar as for regular rows: int32 and
f32 min/max bit-exact, f32 sums within 1e-5 * (sum |f(x)| + |d|), F32_EXACT
inputs bit-exact for every version."""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "flat", "auto"]


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


def descriptors():
    rng = np.random.default_rng(7)
    out = []
    for lens in (
        [5],                                     # one segment
        [0, 0, 3, 0, 1, 0, 0],                   # empties around tiny segments
        [4096] * 3,                              # tile-aligned segments
        [4095, 1, 4097, 8191, 2],                # ends at / around tile boundaries
        [100003],                                # one segment across 25 tiles
        [0] * 5000 + [7] + [0] * 3000,           # many empty segments in one tile
        list(rng.integers(0, 40, 3000)),         # short, ragged
        list(rng.integers(0, 3000, 60)),         # long, ragged
        [1] * 9000,                              # unit segments
        [0] * 10000 + [50000] + [0] * 10000,     # one long segment between runs of empties
        [0] * 4096 + [1] + [0] * 4095 + [2],     # merge-path tiles of ends only
    ):
        lens = np.asarray(lens, np.int64)
        out.append(np.r_[0, np.cumsum(lens)].astype(np.int64))
    out.append(gen.irregular_offsets(9, 4000, 24.0))  # Pareto tail (the bench recipe)
    out.append(gen.irregular_offsets(13, 60000, 1.0))  # the bench's mean-1 mix (mostly empty / unit segments)
    return out


def check(orc, x, off, got, scan, op, f="id", d=None):
    xn = x.cpu().numpy()
    g = got.cpu().numpy()
    if xn.dtype == np.int32 or op in ("min", "max"):
        want = orc.seg_irr(xn, off, scan, op, f, d)
        np.testing.assert_array_equal(g, want.astype(g.dtype))
        return
    want, ab = orc.seg_irr(xn, off, scan, op, f, d, with_absum=True)
    bound = 1e-5 * (ab + (0.0 if d is None else abs(float(d))))
    err = np.abs(g.astype(np.float64) - want)
    assert (err <= bound).all(), f"max err {err.max():.3g} at {err.argmax()}"


def dev(x, misalign):
    if not misalign:
        return x.cuda()
    buf = torch.empty(x.numel() + 1, dtype=x.dtype, device="cuda")
    xd = buf[1:]
    xd.copy_(x)
    return xd


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
def test_irr_descriptors(ifl, orc, version, scan):
    fn = ifl.segscan_irr if scan else ifl.segred_irr
    for k, off in enumerate(descriptors()):
        total = int(off[-1])
        offd = torch.from_numpy(off).cuda()
        for mis in (False, True):
            xi = gen.generate("I32_FULL", 70 + k, total)
            check(orc, xi, off, fn(dev(xi, mis), offd, "sum", version=version), scan, "sum")
            xf = gen.generate("F32_SIGNED", 80 + k, total)
            check(orc, xf, off, fn(dev(xf, mis), offd, "sum", version=version), scan, "sum")


@pytest.mark.parametrize("version", VERS)
def test_irr_scan_in_place(ifl, orc, version):
    """ifl.h: out == in is allowed for the irregular scan (every version)."""
    for k, off in enumerate(descriptors()):
        total = int(off[-1])
        offd = torch.from_numpy(off).cuda()
        for name, dtn in (("I32_FULL", 100), ("F32_SIGNED", 110)):
            x = gen.generate(name, dtn + k, total)
            xd = x.cuda()
            got = ifl.segscan_irr(xd, offd, "sum", version=version, out=xd)
            assert got.data_ptr() == xd.data_ptr()
            check(orc, x, off, got, True, "sum")


@pytest.mark.parametrize("version", VERS)
def test_irr_ops_maps_neutral(ifl, orc, version):
    off = descriptors()[3]
    offd = torch.from_numpy(off).cuda()
    total = int(off[-1])
    xi = gen.generate("I32_FULL", 90, total)
    xf = gen.generate("F32_SIGNED", 91, total)
    for scan in (False, True):
        fn = ifl.segscan_irr if scan else ifl.segred_irr
        for op in ("sum", "prod", "min", "max", "and", "or", "xor"):
            check(orc, xi, off, fn(xi.cuda(), offd, op, "sq", ne=3, version=version), scan, op, "sq", 3)
        for op in ("sum", "min", "max"):
            check(orc, xf, off, fn(xf.cuda(), offd, op, "abs", ne=0.5, version=version), scan, op, "abs", 0.5)


def test_irr_exact_and_regular(ifl, orc):
    off = gen.irregular_offsets(11, 20000, 40.0)
    offd = torch.from_numpy(off).cuda()
    x = gen.generate("F32_EXACT", 92, int(off[-1]))
    for scan in (False, True):
        want = orc.seg_irr(x.numpy(), off, scan).astype(np.float32)
        for v in VERS:
            got = (ifl.segscan_irr if scan else ifl.segred_irr)(x.cuda(), offd, version=v).cpu().numpy()
            np.testing.assert_array_equal(got, want)
    # a regular descriptor reproduces the regular segred / segscan
    xr = gen.matrix("I32_FULL", 93, 300, 77).cuda()
    offr = (torch.arange(301, dtype=torch.int64) * 77).cuda()
    for v in VERS:
        assert torch.equal(ifl.segred_irr(xr.view(-1), offr, "xor", version=v), ifl.segred(xr, "xor"))
        assert torch.equal(ifl.segscan_irr(xr.view(-1), offr, version=v), ifl.segscan(xr).view(-1))


def test_irr_empty_inspector_and_guard(ifl):
    offd = torch.zeros(6, dtype=torch.int64, device="cuda")  # 5 empty segments, no data
    x = torch.empty(0, dtype=torch.int32, device="cuda")
    assert ifl.segred_irr(x, offd, "min").cpu().tolist() == [2**31 - 1] * 5
    assert ifl.segscan_irr(x, offd).numel() == 0
    off = torch.tensor([0, 3, 3, 10, 11], dtype=torch.int64, device="cuda")
    assert ifl.irr_inspect(off, 11) == 7
    with pytest.raises(ifl.IflError):
        ifl.irr_inspect(torch.tensor([0, 5, 3, 11], dtype=torch.int64, device="cuda"), 11)
    with pytest.raises(ifl.IflError):
        ifl.irr_inspect(off, 12)  # off[n] != total
    # the imbalance measure in the guard: Par_top = total / max_len
    ifl.set_thresholds("segred.irr", 1000, 10**9)
    try:
        assert ifl.select("segred.irr", 4000, 64000, 16).version == "top"     # balanced: 4000 >= 1000
        c = ifl.select("segred.irr", 4000, 64000, 6400)                      # skewed: 10 < 1000
        assert c.version == "flat" and c.par_top == 10
    finally:
        ifl.reset_thresholds()


@pytest.mark.parametrize("mean", [1.0, 64.0, 65536.0])
def test_irr_bench_size_sampled(ifl, orc, mean):
    # the bench recipe at 2^26 elements: Pareto lengths, means 1 (mostly empty
    # and unit segments), 64 and 65536 (tiles inside one segment): every
    # output against the oracle, both operations, the merge-path V_FLAT and AUTO
    off = gen.irregular_offsets(12, int((1 << 26) // mean), mean)
    offd = torch.from_numpy(off).cuda()
    x = gen.generate("F32_UNIT", 94, int(off[-1]))
    mx = ifl.irr_inspect(offd, int(off[-1]))
    assert mx == int(np.diff(off).max())
    xd = x.cuda()
    for scan in (False, True):
        want, ab = orc.seg_irr(x.numpy(), off, scan, with_absum=True)
        fn = ifl.segscan_irr if scan else ifl.segred_irr
        for v in (("middle", "flat", "auto") if mean == 64.0 and not scan else ("flat", "auto")):
            got = fn(xd, offd, version=v, max_len=mx).cpu().numpy()
            assert (np.abs(got - want) <= 1e-5 * ab).all(), (v, scan)
    # in place at full size (every tile reads its elements before any tile writes them back)
    xin = x.cuda()
    got = ifl.segscan_irr(xin, offd, version="flat", out=xin)
    assert got.data_ptr() == xin.data_ptr()
    want, ab = orc.seg_irr(x.numpy(), off, True, with_absum=True)
    assert (np.abs(got.cpu().numpy() - want) <= 1e-5 * ab).all(), "in place"
