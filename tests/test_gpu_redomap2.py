"""GPU parity for redomap2 (P:122 map-map-redomap contraction), every
version x dtype x B layout, against the CPU oracle.  Bound:
|C - C*| <= 1e-5 * sum_k |A_ik * Y_kj| + 1e-30 (bf16 products are exact in
f32, so both dtypes share it)."""
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


def bits(t):
    return t.contiguous().view(torch.int16).numpy().view(np.uint16)


def operands(dt, n, m, p, seed=6):
    if dt == "f32":
        A = gen.matrix("F32_SIGNED", seed, n, m)
        Bt = gen.matrix("F32_SIGNED", seed + 1, p, m)
    else:
        A = gen.matrix("BF16_SIGNED", seed, n, m)
        Bt = gen.matrix("BF16_SIGNED", seed + 1, p, m)
    return A, Bt


def check(orc, A, Bt, C):
    a = A.numpy() if A.dtype == torch.float32 else bits(A)
    b = Bt.numpy() if Bt.dtype == torch.float32 else bits(Bt)
    want, ab = orc.redomap2(a, b, b_kmajor=True, with_abs=True)
    err = np.abs(C.cpu().numpy().astype(np.float64) - want)
    bound = 1e-5 * ab + 1e-30
    assert (err <= bound).all(), f"max err {err.max():.3g} at {np.unravel_index(err.argmax(), err.shape)}"


SHAPES = [(1, 1, 1), (3, 5, 7), (1, 1 << 16, 1), (2, 100003, 3), (130, 77, 260), (256, 512, 256),
          (129, 200, 257), (1000, 64, 300), (64, 4096, 1)]


@pytest.mark.parametrize("version", ["top", "middle", "flat", "auto"])
@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_redomap2_versions(ifl, orc, version, dt):
    for (n, m, p) in SHAPES:
        A, Bt = operands(dt, n, m, p)
        C = ifl.redomap2(A.cuda(), Bt.cuda(), b_kmajor=True, version=version)
        check(orc, A, Bt, C)


@pytest.mark.parametrize("version", ["top", "middle", "flat"])
@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_redomap2_row_major_B(ifl, orc, version, dt):
    """B given as yss [m][p] (b_kmajor = 0): same result."""
    # the SIMT tile kernels read yss in place (R24): 32x32 / 128x128 TOP tiles,
    # FLAT's split-K 32x32 tiles, vector and scalar (p % 4 != 0) row loads
    for (n, m, p) in [(5, 33, 17), (200, 128, 300), (1, 5000, 2), (100, 300, 72), (1280, 32, 1280),
                      (1100, 40, 1030), (64, 4096, 64)]:
        A, Bt = operands(dt, n, m, p, seed=9)
        B = Bt.t().contiguous()
        C = ifl.redomap2(A.cuda(), B.cuda(), b_kmajor=False, version=version)
        check(orc, A, Bt, C)


def test_redomap2_closed_forms(ifl):
    # A = 1, B = 1 -> C = m ; A = I -> C = B  (all versions, both dtypes)
    for dt in (torch.float32, torch.bfloat16):
        for v in ("top", "middle", "flat"):
            n, m, p = 130, 264, 300
            C = ifl.redomap2(torch.ones(n, m, dtype=dt, device="cuda"), torch.ones(p, m, dtype=dt, device="cuda"),
                             version=v)
            assert torch.equal(C, torch.full((n, p), float(m), device="cuda"))
            I = torch.eye(m, dtype=dt, device="cuda")
            Bt = gen.matrix("BF16_SIGNED", 3, p, m).to(dt).cuda()
            C = ifl.redomap2(I, Bt, version=v)
            assert torch.equal(C, Bt.t().float()), (dt, v)


@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_config2_family_k20(ifl, orc, dt):
    """BASELINE.json configs[2]: A[2^a][2^(k-2a)] x B[2^(k-2a)][2^a], k = 20,
    tall-skinny to square, every version."""
    k = 20
    for a in range(0, k // 2 + 1, 2):
        n = p = 1 << a
        m = 1 << (k - 2 * a)
        A, Bt = operands(dt, n, m, p, seed=6)
        for v in ("top", "middle", "flat", "auto"):
            C = ifl.redomap2(A.cuda(), Bt.cuda(), version=v)
            check(orc, A, Bt, C)


def test_tc_dense_square(ifl, orc):
    """Dense bf16 square through the tcgen05 kernel, sampled rows vs oracle."""
    n = m = p = 1024
    A, Bt = operands("bf16", n, m, p, seed=11)
    C = ifl.redomap2(A.cuda(), Bt.cuda(), version="top")
    rows = [0, 1, 127, 128, 511, 1023]
    check(orc, A[rows], Bt, C[rows])
    # B as yss [m][p]: the tcgen05 kernel reads it MN-major in place (R24),
    # TOP and the split-K FLAT tiles; ragged p (a partial 64-column box)
    for (nn, mm, pp) in [(1024, 1024, 1024), (300, 640, 328), (200, 128, 8), (130, 72, 24)]:
        A2, Bt2 = operands("bf16", nn, mm, pp, seed=12)
        B2 = Bt2.t().contiguous().cuda()
        for v in ("top", "flat"):
            C2 = ifl.redomap2(A2.cuda(), B2, b_kmajor=False, version=v)
            r2 = sorted({0, 1, 127, 128, nn - 1})
            check(orc, A2[r2], Bt2, C2[r2])


# ------------------------------------------ row-level leaves of the matmul tree (NEXT-2)

ROW_SHAPES = [(1, 1, 1), (3, 5, 7), (1000, 64, 3), (130, 77, 260), (7, 8192, 5), (64, 1000, 1), (4096, 16, 16)]


@pytest.mark.parametrize("version", ["row_top", "row_middle"])
@pytest.mark.parametrize("dt", ["f32", "bf16"])
@pytest.mark.parametrize("kmajor", [True, False])
def test_redomap2_row_versions(ifl, orc, version, dt, kmajor):
    tdt = torch.float32 if dt == "f32" else torch.bfloat16
    for (n, m, p) in ROW_SHAPES:
        A, Bt = operands(dt, n, m, p, seed=21)
        A, Bt = A.to(tdt), Bt.to(tdt)
        B = Bt if kmajor else Bt.t().contiguous()
        C = ifl.redomap2(A.cuda(), B.cuda(), b_kmajor=kmajor, version=version)
        check(orc, A, Bt, C)


def test_redomap2_row_middle_notfit_and_tree(ifl, orc):
    A, Bt = operands("f32", 3, 9000, 2)
    with pytest.raises(ifl.IflError) as e:
        ifl.redomap2(A.cuda(), Bt.cuda(), version="row_middle")
    assert e.value.code == ifl.IFL_ENOTFIT
    # the 5-leaf tree tuner: times every leaf, installs the row and the two-map thresholds
    try:
        train = [(1 << a, 1 << (18 - 2 * a), 1 << a) for a in range(0, 10)]
        t_top, t_intra, tbl = ifl.tune("redomap2.f32.tree", train, reps=2, cost=1)
        assert tbl.shape == (len(train), 5) and np.isfinite(tbl[:, 2:]).all()
        assert ifl.get_thresholds("redomap2.f32") == (t_top, t_intra)
        rt, ri = ifl.get_thresholds("redomap2.f32.row")
        for (n, m, p) in train[:4]:
            A, Bt = operands("f32", n, m, p, seed=22)
            C, ch = ifl.redomap2(A.cuda(), Bt.cuda(), return_choice=True)
            check(orc, A, Bt, C)
            assert ch.version in ("row_top", "row_middle", "top", "middle", "flat")
    finally:
        ifl.reset_thresholds()


SKINNY = [(1, 1, 1), (1, 4096, 1), (3, 1000003, 5), (8, 1 << 20, 8), (7, 5000, 3), (16, 300001, 16), (5, 64, 40),
          (64, 20000, 64), (1, 1 << 22, 2), (33, 9999, 2)]


@pytest.mark.parametrize("dt", ["f32", "bf16"])
@pytest.mark.parametrize("kmajor", [True, False])
def test_flat_skinny_engine(ifl, orc, dt, kmajor):
    """V_FLAT's split-K register-block engine (n*p <= 4096 f32 / <= 256 bf16):
    both B layouts read in place (no transposition), odd n and p (partial
    register tiles), m not a multiple of the vector width, misaligned
    operands (the scalar form), and k split across many CTAs."""
    tdt = torch.float32 if dt == "f32" else torch.bfloat16
    for (n, m, p) in SKINNY:
        A, Bt = operands(dt, n, m, p, seed=40)
        A, Bt = A.to(tdt), Bt.to(tdt)
        B = Bt if kmajor else Bt.t().contiguous()
        C = ifl.redomap2(A.cuda(), B.cuda(), b_kmajor=kmajor, version="flat")
        check(orc, A, Bt, C)
        # misaligned A (offset by one element): scalar engine
        buf = torch.empty(n * m + 1, dtype=tdt, device="cuda")
        Am = buf[1:].view(n, m)
        Am.copy_(A.cuda())
        C2 = ifl.redomap2(Am, B.cuda(), b_kmajor=kmajor, version="flat")
        check(orc, A, Bt, C2)


@pytest.mark.parametrize("dt", ["f32", "bf16"])
def test_flat_skinny_last_cta_finalize(ifl, dt):
    """The skinny engine is one kernel: the last CTA of each output tile sums
    the k-splits' partials in split order (deterministic) and re-arms its
    arrival counter, so one workspace serves repeated and differently shaped
    calls (graph replays included) with bit-identical results."""
    tdt = torch.float32 if dt == "f32" else torch.bfloat16
    ws = ifl.workspace(ifl.workspace_bytes("redomap2", 64, 1 << 20, 64, dt), "cuda", "skinny_fin_" + dt)
    ref = {}
    for rep in range(3):
        for (n, m, p) in [(8, 1 << 20, 8), (3, 1000003, 5), (16, 300001, 16), (64, 20000, 64)]:
            if dt == "bf16" and n * p > 256:
                continue
            A, Bt = operands(dt, n, m, p, seed=41)
            A, Bt = A.to(tdt).cuda(), Bt.to(tdt).cuda()
            C = ifl.redomap2(A, Bt, version="flat", ws=ws)
            if rep == 0:
                ref[(n, m, p)] = C.clone()
                # a fresh workspace gives the same result bit for bit
                assert torch.equal(C, ifl.redomap2(A, Bt, version="flat"))
            else:
                assert torch.equal(C, ref[(n, m, p)])
    torch.cuda.synchronize()
    # the arrival counters (the workspace's first 16 KB) are back at zero
    assert int(ws[:16384].sum().item()) == 0
