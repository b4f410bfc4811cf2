"""GPU parity at the sizes the bench and BASELINE.json name, beyond what the
oracle finishes in seconds: sampled outputs against the oracle one by one,
plus properties that hold at any size (64-bit indexing past 2^31
elements; configs[4]'s 2^30-element reduce through the device-level split of
dist.py; the 8192^3 tcgen05 contraction, rows and columns of the first and
last tiles).  int32 and min/max bit-exact; f32 sums within 1e-5 * sum|f(x)|."""
import os
import socket

import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


def _want(orc, xv, rows, scan, dt):
    xs = xv[rows].cpu().numpy()
    if dt == "i32":
        return (orc.segscan(xs, "sum") if scan else orc.segred(xs, "sum")), None
    return (orc.segscan if scan else orc.segred)(xs, "sum", with_absum=True)


def _rows_check(want, got, rows, dt, what=""):
    g = got[rows].cpu().numpy()
    w, ab = want
    if dt == "i32":
        np.testing.assert_array_equal(g, w, err_msg=what)
    else:
        err = np.abs(g.astype(np.float64) - w)
        bad = err > 1e-5 * ab
        assert not bad.any(), f"{what}: max err {err.max():.4g} (bound {(1e-5 * ab)[bad][:3]}) at {np.argwhere(bad)[:3]}"


# n*m = 2^31 + small: every flat index above 2^31 must be addressed in 64 bits
BIG = [(5, 429496730), (65537, 32768)]


@pytest.mark.parametrize("dt", ["i32", "f32"])
@pytest.mark.parametrize("scan", [False, True])
def test_over_2_31_elements(ifl, orc, dt, scan):
    name = "I32_FULL" if dt == "i32" else "F32_UNIT"
    for (n, m) in BIG:
        N = n * m
        assert N > 2**31
        x = gen.generate(name, 12, N, device="cuda")
        xv = x.view(n, m)
        out = torch.empty((n, m) if scan else (n,), dtype=x.dtype, device="cuda")
        rows = sorted({0, 1, n // 2, n - 2, n - 1})
        want = _want(orc, xv, rows, scan, dt)
        for v in ("top", "middle", "flat", "auto"):
            if v == "top" and scan and m > 1 << 24:
                continue  # one thread walking 4 x 10^8 elements of a scan: minutes, nothing new
            fn = ifl.segscan if scan else ifl.segred
            got = fn(xv, "sum", version=v, out=out)
            torch.cuda.synchronize()
            _rows_check(want, got, rows, dt, f"{v} n={n} m={m}")
        del x, xv, out
        torch.cuda.empty_cache()


def test_over_2_31_rows(ifl):
    """n = 2^31 + 5 rows of one element: out[i] = d (+) f(x[i]) for every i --
    checked on the whole array against a torch expression of that closed form."""
    n = 2**31 + 5
    x = gen.generate("I32_SMALL", 13, n, device="cuda")
    for v in ("top", "middle", "flat", "auto"):
        got = ifl.segred(x.view(n, 1), "sum", ne=7, version=v)
        assert torch.equal(got, x + 7), v
        del got
        got = ifl.segscan(x.view(n, 1), "max", ne=0, version=v)
        assert torch.equal(got.view(-1), torch.clamp(x, min=0)), v
        del got
        torch.cuda.empty_cache()


@pytest.mark.parametrize("dt", ["i32", "f32"])
def test_irregular_over_2_31_elements(ifl, orc, dt):
    """Irregular segments over 2^31 + 5 elements through the merge-path V_FLAT
    (64-bit element and tile coordinates): 40 segments of ragged lengths with
    empty ones between them, one of them holding element 2^31; sampled
    segments (first, last, the one across 2^31, two more) against the oracle,
    both operations."""
    name = "I32_FULL" if dt == "i32" else "F32_UNIT"
    total = 2**31 + 5
    rng = np.random.default_rng(21)
    w = rng.uniform(0.2, 1.8, 40)
    lens = np.floor(w / w.sum() * total).astype(np.int64)
    lens[-1] += total - lens.sum()
    lens = np.insert(lens, [3, 3, 17, 30], 0)  # empty segments
    off = np.zeros(lens.size + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    assert off[-1] == total
    x = gen.generate(name, 14, total, device="cuda")
    offd = torch.from_numpy(off).cuda()
    cross = int(np.searchsorted(off, 2**31, side="right") - 1)
    segs = sorted({0, 3, cross, 25, lens.size - 1})
    for scan in (False, True):
        fn = ifl.segscan_irr if scan else ifl.segred_irr
        got = fn(x, offd, "sum", version="flat")
        torch.cuda.synchronize()
        for i in segs:
            a, b = int(off[i]), int(off[i + 1])
            xs = x[a:b].cpu().numpy()
            sub = np.array([0, b - a], np.int64)
            if dt == "i32":
                want = orc.seg_irr(xs, sub, scan)
                g = got[a:b] if scan else got[i:i + 1]
                np.testing.assert_array_equal(g.cpu().numpy(), want, err_msg=f"seg {i} scan={scan}")
            else:
                want, ab = orc.seg_irr(xs, sub, scan, with_absum=True)
                g = (got[a:b] if scan else got[i:i + 1]).cpu().numpy().astype(np.float64)
                assert (np.abs(g - want) <= 1e-5 * ab).all(), f"seg {i} scan={scan}"
        del got
        torch.cuda.empty_cache()
    del x
    torch.cuda.empty_cache()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_config4_2_30_through_dist(ifl, orc):
    """configs[4]: the 2^30-element segmented reduce through dist.segred_dist
    (NCCL world 1: the outer plan and the inner plan with its all_reduce) and
    through G = 8 virtual shards of either split combined by the library's own
    kernels, for n in {1, 2^4, 2^10, 2^16, 2^20, 2^24},
    int32 bit-exact on sampled rows (and on every row for n >= 2^16 against
    the row-split result)."""
    import torch.distributed as td
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    N = 1 << 30
    x = gen.generate("I32_FULL", 8, N, device="cuda")
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        for k in (0, 4, 10, 16, 20, 24):
            n, m = 1 << k, N >> k
            xv = x.view(n, m)
            rows = sorted({0, n // 3, n - 1})
            want = orc.segred(xv[rows].cpu().numpy(), "sum", "id", 5)
            outs = []
            for t_dev in (1, n + 1):  # outer plan (n >= t_dev) / inner plan
                plan = dist.plan_segred(n, m, 1, 0, t_dev)
                out = dist.segred_dist(xv, n, m, "sum", "id", 5, plan=plan, gather=True)
                np.testing.assert_array_equal(out[rows].cpu().numpy(), want)
                outs.append(out)
            assert torch.equal(outs[0], outs[1])
            G = 8
            if n >= G:  # row shards (outer split), concatenated
                per = n // G
                sh = torch.cat([ifl.segred(xv[r * per:(r + 1) * per], "sum", ne=5) for r in range(G)])
                assert torch.equal(sh, outs[0])
            cuts = [(m * r) // G for r in range(G + 1)]  # column shards (inner split), partials without d
            parts = torch.stack([ifl.segred(xv[:, cuts[r]:cuts[r + 1]].contiguous(), "sum") for r in range(G)], 1)
            total = ifl.segred(parts.contiguous(), "sum", ne=5)
            assert torch.equal(total, outs[0])
            del parts, total, outs
    finally:
        td.destroy_process_group()


def test_tc_8192_cube_first_last_tiles(ifl, orc):
    """The reported dense shape, 8192^3 bf16 through the tcgen05 kernel:
    full rows of C from the first and last 128-row tiles and full columns from
    the first and last 256-column tiles against the oracle."""
    n = m = p = 8192
    A = gen.matrix("BF16_SIGNED", 31, n, m)
    Bt = gen.matrix("BF16_SIGNED", 32, p, m)
    C = ifl.redomap2(A.cuda(), Bt.cuda(), version="top").cpu()

    def bits(t):
        return t.contiguous().view(torch.int16).numpy().view(np.uint16)

    rows = [0, 1, 127, 128, 8063, 8064, 8191]
    want, ab = orc.redomap2(bits(A[rows]), bits(Bt), b_kmajor=True, with_abs=True)
    assert (np.abs(C[rows].numpy().astype(np.float64) - want) <= 1e-5 * ab + 1e-30).all()
    cols = [0, 255, 256, 7935, 7936, 8191]
    want, ab = orc.redomap2(bits(A), bits(Bt[cols]), b_kmajor=True, with_abs=True)
    assert (np.abs(C[:, cols].numpy().astype(np.float64) - want) <= 1e-5 * ab + 1e-30).all()
    # B as yss [m][p] (b_kmajor = 0): the MN-major operand path, no transposition
    C2 = ifl.redomap2(A.cuda(), Bt.t().contiguous().cuda(), b_kmajor=False, version="top").cpu()
    rows2 = [0, 8064, 8191]
    want, ab = orc.redomap2(bits(A[rows2]), bits(Bt), b_kmajor=True, with_abs=True)
    assert (np.abs(C2[rows2].numpy().astype(np.float64) - want) <= 1e-5 * ab + 1e-30).all()
    want, ab = orc.redomap2(bits(A), bits(Bt[[0, 7936, 8191]]), b_kmajor=True, with_abs=True)
    assert (np.abs(C2[:, [0, 7936, 8191]].numpy().astype(np.float64) - want) <= 1e-5 * ab + 1e-30).all()
