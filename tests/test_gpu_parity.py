"""GPU parity: every version of segred / segscan (through the C ABI, via the
thin binding) against the CPU oracle on the same seeded inputs.

Bar: int32 ops and f32 min/max bit-exact; f32 sums
within 1e-5 * sum|f(x)| (the C3 bound); f32 prod within m * 2^-23 relative;
F32_EXACT inputs bit-exact for every version and every op.
"""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "cluster", "flat", "auto"]
TINY = [0, 1, 2, 3, 5, 8, 31, 32, 33, 127, 1024, 4097]


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


def make(dist, seed, n, m, dev="cuda", misalign=False):
    x = gen.matrix(dist, seed, n, m)
    if dist == "F32_PROD":
        pass
    if misalign:
        buf = torch.empty(n * m + 1, dtype=x.dtype, device=dev)
        xd = buf[1:].view(n, m)
        xd.copy_(x)
        return x, xd
    return x, x.to(dev)


def gen_for(op, dt, seed, n, m, misalign=False):
    if dt == "i32":
        return make("I32_SMALL" if op == "prod" else "I32_FULL", seed, n, m, misalign=misalign)
    if op == "prod":
        x = (0.5 + gen.matrix("F32_UNIT", seed, n, m)).contiguous()
        return x, x.cuda()
    return make("F32_SIGNED", seed, n, m, misalign=misalign)


def assert_parity(orc, x, got, scan, op, f, d, dt):
    xn = x.cpu().numpy()
    g = got.cpu().numpy()
    if dt == "i32":
        want = orc.segscan(xn, op, f, d) if scan else orc.segred(xn, op, f, d)
        np.testing.assert_array_equal(g, want)
        return
    if scan:
        want, ab = orc.segscan(xn, op, f, d, with_absum=True)
    else:
        want, ab = orc.segred(xn, op, f, d, with_absum=True)
    if op in ("min", "max"):
        np.testing.assert_array_equal(g, want.astype(np.float32))
    elif op == "sum":
        dd = 0.0 if d is None else abs(float(d))
        err = np.abs(g.astype(np.float64) - want)
        bound = 1e-5 * (ab + dd)
        bad = err > bound
        assert not bad.any(), f"max err {err.max()} bound {bound[bad][:4]} at {np.argwhere(bad)[:4]}"
    else:  # prod
        m = xn.shape[1]
        err = np.abs(g.astype(np.float64) - want)
        assert (err <= (m + 2) * 2.0**-23 * np.abs(want) + 1e-30).all()


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("dt", ["i32", "f32"])
@pytest.mark.parametrize("scan", [False, True])
def test_tiny_grid_sum(ifl, orc, version, dt, scan):
    """All (n, m) on the tiny grid, sum/id: spans ragged tails and empties."""
    for n in TINY:
        for m in TINY:
            if n * m > 1 << 20:
                continue
            x, xd = gen_for("sum", dt, 1, n, m)
            fn = ifl.segscan if scan else ifl.segred
            got = fn(xd, "sum", "id", version=version)
            assert_parity(orc, x, got, scan, "sum", "id", None, dt)


OPS_I = ["sum", "prod", "min", "max", "and", "or", "xor"]
OPS_F = ["sum", "prod", "min", "max"]
SHAPES = [(1, 1), (3, 7), (64, 33), (300, 4), (5, 7169), (2, 20000), (1000, 64), (33, 1000)]


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
@pytest.mark.parametrize("f", ["id", "sq", "abs"])
def test_ops_maps(ifl, orc, version, scan, f):
    fn = ifl.segscan if scan else ifl.segred
    for dt, ops in (("i32", OPS_I), ("f32", OPS_F)):
        for op in ops:
            for (n, m) in SHAPES:
                x, xd = gen_for(op, dt, 2, n, m)
                got = fn(xd, op, f, version=version)
                assert_parity(orc, x, got, scan, op, f, None, dt)


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
def test_neutral_element_applied_once(ifl, orc, version, scan):
    fn = ifl.segscan if scan else ifl.segred
    for (n, m) in [(4, 0), (5, 1), (17, 999), (3, 7168 * 2 + 5)]:
        x, xd = gen_for("sum", "i32", 3, n, m)
        for op, d in (("sum", 12345), ("min", -7), ("xor", 0x5A5A), ("prod", 3)):
            got = fn(xd, op, "id", ne=d, version=version)
            assert_parity(orc, x, got, scan, op, "id", d, "i32")
        xf, xfd = gen_for("sum", "f32", 3, n, m)
        got = fn(xfd, "sum", "id", ne=2.5, version=version)
        assert_parity(orc, xf, got, scan, "sum", "id", 2.5, "f32")


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
def test_misaligned_and_odd(ifl, orc, version, scan):
    """Base pointer offset by 4 bytes, odd m: row starts not 16-byte aligned."""
    fn = ifl.segscan if scan else ifl.segred
    for (n, m) in [(7, 5), (33, 1350), (1024, 31), (3, 50001), (1, 855280 // 8)]:
        for dt in ("i32", "f32"):
            x, xd = gen_for("sum", dt, 4, n, m, misalign=True)
            assert xd.data_ptr() % 16 != 0
            if scan:
                ob = torch.empty(n * m + 1, dtype=xd.dtype, device="cuda")[1:].view(n, m)
                got = fn(xd, "sum", "id", version=version, out=ob)
            else:
                got = fn(xd, "sum", "id", version=version)
            assert_parity(orc, x, got, scan, "sum", "id", None, dt)


@pytest.mark.parametrize("version", ["top", "middle", "flat"])
def test_inplace_scan(ifl, orc, version):
    # (100, 1024) / (7, 5120): tile-aligned segments (single-pass engine);
    # (3, 2^20) / (1, 5120*50+3): segments across tiles (job-ring engine)
    for (n, m) in [(100, 100), (2, 7168 * 3 + 1), (4096, 8), (100, 1024), (7, 5120), (3, 1 << 20),
                   (1, 5120 * 50 + 3)]:
        x, xd = gen_for("sum", "i32", 5, n, m)
        got = ifl.segscan(xd, "sum", "id", version=version, out=xd)
        assert got.data_ptr() == xd.data_ptr()
        assert_parity(orc, x, got, True, "sum", "id", None, "i32")


@pytest.mark.parametrize("scan", [False, True])
def test_f32_exact_all_versions_bitwise(ifl, orc, scan):
    """F32_EXACT: every association is exact, so all versions agree bit for
    bit with each other and with the oracle, even for sum/scan."""
    fn = ifl.segscan if scan else ifl.segred
    for (n, m) in [(1, 1 << 20), (64, 4096), (4096, 64), (1 << 16, 3)]:
        x, xd = make("F32_EXACT", 3, n, m)
        want = (orc.segscan if scan else orc.segred)(x.numpy(), "sum")
        for v in VERS:
            if v == "cluster" and scan and m > 16 * 40960:
                continue  # a cluster-per-row scan does not fit rows this long (IFL_ENOTFIT, test_cluster_level)
            got = fn(xd, "sum", "id", version=v).cpu().numpy()
            np.testing.assert_array_equal(got, want.astype(np.float32), err_msg=v)


def test_flat_many_tiles_lookback(ifl, orc):
    """Long segments spanning many flat tiles (decoupled look-back chains)
    and repeated calls on one workspace (epoch re-arming)."""
    for (n, m) in [(1, 7168 * 200 + 3), (3, 1 << 20), (7, 7168 - 1), (2, 7168 + 1)]:
        for dt in ("i32", "f32"):
            x, xd = gen_for("sum", dt, 6, n, m)
            for _ in range(3):
                assert_parity(orc, x, ifl.segred(xd, "sum", version="flat"), False, "sum", "id", None, dt)
                assert_parity(orc, x, ifl.segscan(xd, "sum", version="flat"), True, "sum", "id", None, dt)


@pytest.mark.parametrize("dt", ["i32", "f32"])
def test_workspace_shared_after_segred(ifl, orc, dt):
    """a segred on N1 elements leaves small-integer partials where a
    later segscan on N2 > 8 N1 elements keeps its status words.  The status
    tag is a scrambled epoch, so stale partials are not taken for valid words;
    the binding also keys its cached workspaces by entry point."""
    ws = torch.zeros(ifl.workspace_bytes("segscan", 1, 1 << 22), dtype=torch.uint8, device="cuda")
    small = torch.ones(64, 5121, dtype=torch.int32 if dt == "i32" else torch.float32, device="cuda")
    for _ in range(3):
        ifl.segred(small * 2, "sum", version="flat", ws=ws)  # partials 2, 4, ... 10242
        for (n, m) in [(1, 1 << 22), (4, 1 << 20), (1000, 4000)]:
            x, xd = gen_for("sum", dt, 8, n, m)
            assert_parity(orc, x, ifl.segscan(xd, "sum", version="flat", ws=ws), True, "sum", "id", None, dt)
            ifl.segred(xd, "sum", version="flat", ws=ws)


def test_config0_int32_1024x1024(ifl, orc):
    """BASELINE.json configs[0]: int32 segmented sum 1024 x 1024, bit-exact,
    plus the closed form x[i][j] = i*m + j -> m^2 i + m(m-1)/2."""
    n = m = 1024
    x, xd = make("I32_FULL", 1, n, m)
    want = orc.segred(x.numpy(), "sum")
    for v in VERS:
        np.testing.assert_array_equal(ifl.segred(xd, "sum", version=v).cpu().numpy(), want)
    idx = (torch.arange(n, dtype=torch.int64)[:, None] * m + torch.arange(m)).to(torch.int32).cuda()
    cf = m * m * np.arange(n, dtype=np.int64) + m * (m - 1) // 2
    for v in VERS:
        np.testing.assert_array_equal(ifl.segred(idx, "sum", version=v).cpu().numpy(), cf)


@pytest.mark.slow
@pytest.mark.parametrize("scan", [False, True])
def test_config1_sweep_full_size_sampled(ifl, orc, scan):
    """BASELINE.json configs[1]: n*m = 2^26, n = 2^k.  Every version at full
    size; sampled rows against the oracle (F32_UNIT, sum and sq)."""
    N = 1 << 26
    x = gen.generate("F32_UNIT", 2, N, device="cuda")
    fn = ifl.segscan if scan else ifl.segred
    for k in range(0, 27, 2):
        n, m = 1 << k, 1 << (26 - k)
        xv = x.view(n, m)
        rows = sorted(set([0, n - 1, n // 2] + list(range(0, n, max(1, n // 5)))))[:8]
        xs = xv[rows].cpu()
        for f in ("id", "sq"):
            for v in (["top", "middle", "flat", "auto"] if k >= 4 or not scan else ["middle", "flat", "auto"]):
                got = fn(xv, "sum", f, version=v)
                assert_parity(orc, xs, got[rows], scan, "sum", f, None, "f32")
        del xv


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("scan", [False, True])
def test_small_m_kernels(ifl, orc, version, scan):
    """Row lengths with dedicated TOP kernels (m in {1,2,4}: packed words;
    {8,16}: thread-per-row registers; {16,32,64}: warp tiles via shared memory),
    ragged row counts (partial warps / CTAs), every op, int32 and f32."""
    fn = ifl.segscan if scan else ifl.segred
    for m in (1, 2, 4, 8, 16, 32, 64):
        for n in (1, 31, 33, 257, 4099):
            for dt, ops in (("i32", OPS_I), ("f32", OPS_F)):
                for op in ops:
                    x, xd = gen_for(op, dt, 5, n, m)
                    got = fn(xd, op, "sq" if op == "sum" else "id", version=version)
                    assert_parity(orc, x, got, scan, op, "sq" if op == "sum" else "id", None, dt)


@pytest.mark.parametrize("version", ["flat", "middle"])
@pytest.mark.parametrize("dt", ["i32", "f32"])
def test_segred_long_rows_split_and_cluster(ifl, orc, dt, version):
    # rows >= 8192 elements: V_FLAT uniform row pieces + per-row combine; V_MIDDLE
    # one 512/1024-thread CTA per row, or a thread-block cluster per row with a
    # DSMEM combine when there are fewer rows than SMs
    for (n, m, mis) in [(1, (1 << 20) + 5, True), (3, (1 << 16) + 13, False), (7, 1 << 17, True),
                        (130, 1 << 16, False), (300, 8200, True), (64, 1 << 15, False)]:
        for op in (["sum", "min", "xor", "prod"] if dt == "i32" else ["sum", "max"]):
            x, xd = gen_for(op, dt, 17, n, m, misalign=mis)
            got = ifl.segred(xd, op, "sq" if op != "prod" else "id", ne=(2 if dt == "i32" else 0.5), version=version)
            assert_parity(orc, x, got, False, op, "sq" if op != "prod" else "id", 2 if dt == "i32" else 0.5, dt)


@pytest.mark.parametrize("f", ["id", "sq", "abs"])
def test_middle_aligned_rows(ifl, orc, f):
    """V_MIDDLE's vector kernel (m % 4 == 0, aligned, m <= 16*G): every group
    size G = 1..512 (rows of 4..8188), ragged n, all ops, d applied once."""
    for dt, ops in (("i32", OPS_I), ("f32", OPS_F)):
        for op in ops:
            for (n, m) in [(37, 4), (9, 12), (300, 16), (129, 20), (65, 64), (17, 100), (5, 256),
                           (3, 2048), (7, 4096), (2, 8188)]:
                x, xd = gen_for(op, dt, 5, n, m)
                got = ifl.segred(xd, op, f, version="middle")
                assert_parity(orc, x, got, False, op, f, None, dt)
    x, xd = gen_for("sum", "i32", 6, 11, 4096)
    assert_parity(orc, x, ifl.segred(xd, "max", "abs", ne=-3, version="middle"), False, "max", "abs", -3, "i32")


@pytest.mark.parametrize("version", VERS)
@pytest.mark.parametrize("dt", ["i32", "f32"])
def test_reverse_scan(ifl, orc, version, dt):
    """reverse = 1: out[i][j] = d (+) f(x[i][m-1]) (+) ... (+) f(x[i][j]) (ifl.h),
    every version (TOP / MIDDLE mirror rows, FLAT mirrors the flat index space:
    tile-aligned and job-ring engines), ragged shapes, misaligned and in place."""
    shapes = [(1, 1), (5, 3), (33, 64), (7, 1000), (3, 5120), (2, 50001), (200, 1024), (1, 5120 * 13 + 7)]
    ops = OPS_I if dt == "i32" else OPS_F
    for (n, m) in shapes:
        for op in ops:
            x, xd = gen_for(op, dt, 21, n, m)
            got = ifl.segscan(xd, op, "sq" if op == "sum" else "id", ne=(3 if dt == "i32" else 0.5) if op == "sum" else None,
                              version=version, reverse=True)
            d = (3 if dt == "i32" else 0.5) if op == "sum" else None
            f = "sq" if op == "sum" else "id"
            if dt == "i32":
                np.testing.assert_array_equal(got.cpu().numpy(), orc.segscan(x.numpy(), op, f, d, reverse=True))
            else:
                want, ab = orc.segscan(x.numpy(), op, f, d, reverse=True, with_absum=True)
                g = got.cpu().numpy().astype(np.float64)
                if op in ("min", "max"):
                    np.testing.assert_array_equal(g, want)
                elif op == "sum":
                    assert (np.abs(g - want) <= 1e-5 * (ab + 0.5)).all()
                else:
                    assert (np.abs(g - want) <= (m + 2) * 2.0**-23 * np.abs(want) + 1e-30).all()
        # misaligned input/output and in place
        x, xd = gen_for("sum", dt, 22, n, m, misalign=True)
        want = orc.segscan(x.numpy(), "sum", reverse=True, with_absum=dt == "f32")
        got = ifl.segscan(xd, "sum", version=version, reverse=True)
        got2 = ifl.segscan(xd, "sum", version=version, reverse=True, out=xd)
        for g in (got, got2):
            if dt == "i32":
                np.testing.assert_array_equal(g.cpu().numpy(), want)
            else:
                assert (np.abs(g.cpu().numpy() - want[0]) <= 1e-5 * want[1]).all()


def test_cluster_level(ifl, orc):
    """V_CLUSTER (reading R18): cluster sizes 1..16 across row lengths, a
    segscan row at the fit limit and one past it (IFL_ENOTFIT), and AUTO
    taking the cluster leaf once its threshold is set."""
    for (n, m) in [(1, 16 * 40960), (3, 300007), (8, 1 << 20), (40, 70000), (700, 5000)]:
        for dt in ("i32", "f32"):
            x, xd = gen_for("sum", dt, 31, n, m)
            assert_parity(orc, x, ifl.segred(xd, "sum", "sq", version="cluster"), False, "sum", "sq", None, dt)
            if m > 16 * 40960:
                continue  # segred only: a cluster-per-row scan keeps the row in shared memory
            assert_parity(orc, x, ifl.segscan(xd, "sum", "sq", version="cluster"), True, "sum", "sq", None, dt)
            got = ifl.segscan(xd, "max", version="cluster", reverse=True)
            want = orc.segscan(x.numpy(), "max", reverse=True)
            np.testing.assert_array_equal(got.cpu().numpy(), want.astype(got.cpu().numpy().dtype))
    x, xd = gen_for("sum", "i32", 32, 2, 16 * 40960 + 4)
    with pytest.raises(ifl.IflError) as e:
        ifl.segscan(xd, version="cluster")
    assert e.value.code == ifl.IFL_ENOTFIT
    assert_parity(orc, x, ifl.segred(xd, "sum", version="cluster"), False, "sum", "id", None, "i32")
    try:
        ifl.set_thresholds("segscan.b4", 1 << 40, 1 << 40)
        ifl.set_thresholds("segscan.b4.cl", 1, 1)
        x, xd = gen_for("sum", "f32", 33, 16, 100000)
        got, ch = ifl.segscan(xd, return_choice=True)
        assert ch.version == "cluster"
        assert_parity(orc, x, got, True, "sum", "id", None, "f32")
    finally:
        ifl.reset_thresholds()


def test_middle_group_size_dimension(ifl, orc):
    """Reading R19: V_MIDDLE's group size x 2^shift (shift -3..3, the tuned
    tile/group-size dimension) keeps every result; the tuner site picks one."""
    try:
        for shift in range(-3, 4):
            ifl.set_thresholds("segred.b4.midg", 8 + shift, 0)
            ifl.set_thresholds("segscan.b4.midg", 8 + shift, 0)
            for (n, m) in [(37, 4), (65, 64), (17, 100), (5, 1024), (3, 4096), (9, 3001)]:
                for dt in ("i32", "f32"):
                    x, xd = gen_for("sum", dt, 40, n, m)
                    assert_parity(orc, x, ifl.segred(xd, "sum", version="middle"), False, "sum", "id", None, dt)
                    assert_parity(orc, x, ifl.segscan(xd, "sum", version="middle"), True, "sum", "id", None, dt)
        ifl.reset_thresholds()
        train = [(1 << k, 1 << (20 - k)) for k in range(10, 21, 2)]
        for site in ("segred.b4.midg", "segscan.b4.midg"):
            t, u, tbl = ifl.tune(site, train, reps=2, cost=1)
            assert 6 <= t <= 10 and u == 0 and tbl.shape == (len(train), 5)
            assert ifl.get_thresholds(site) == (t, 0)
    finally:
        ifl.reset_thresholds()
