"""GPU parity for ifl_lvc, the whole LocVolCalib loop of Fig 6a,
against the oracle's numT Thomas solves per site with the state in double.

Bound (derived): each step's solve is within the tridag bar
1e-5 * max(1, ||x||_inf) of the exact solve of its own f32 input, and the
recipe's matrices have row margin |b| - |a| - |c| = 1, so ||A^-1||_inf <= 1
and step errors never grow: after numT steps
    max |x - x*| <= numT * 1e-5 * max(1, ||x*||_inf).
"""
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


def run_and_check(ifl, orc, numS, numT, numX, numY, version, seed=13, sample=None):
    (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(seed, numS, numX, numY)
    xd, yd = xs.cuda(), ys.cuda()
    xc = tuple(t.cuda() for t in (ax, bx, cx))
    yc = tuple(t.cuda() for t in (ay, by, cy))
    ch = ifl.lvc(xd, yd, xc, yc, numT, version=version, return_choice=True)
    torch.cuda.synchronize()
    idx = np.arange(numS) if sample is None else np.asarray(sample)
    co = [t.numpy() for t in (ax, bx, cx, ay, by, cy)]
    want_x, want_y = orc.lvc(*co, xs.numpy()[idx], ys.numpy()[idx], numT)
    for got, want in ((xd.cpu().numpy()[idx], want_x), (yd.cpu().numpy()[idx], want_y)):
        tol = max(numT, 1) * 1e-5 * max(1.0, np.abs(want).max())
        err = np.abs(got.astype(np.float64) - want).max()
        assert err <= tol, f"{version} S={numS} T={numT} X={numX} Y={numY}: err {err:.3g} > {tol:.3g}"
    return ch


SHAPES = [  # (numS, numT, numX, numY)
    (2, 3, 32, 256),    # small's sites, few steps
    (3, 5, 256, 32),    # medium's sites
    (2, 4, 5, 7),       # ragged, G = 1
    (3, 6, 17, 33),     # ragged, non-multiple-of-4 rows (scalar path)
    (2, 3, 300, 9),     # IT = 16 path (L = 300 > 256)
    (1, 2, 1, 1),       # degenerate 1x1 systems
    (4, 1, 64, 64),
]


@pytest.mark.parametrize("version", ["outer", "top", "middle", "flat", "auto"])
def test_lvc_versions(ifl, orc, version):
    for (S, T, X, Y) in SHAPES:
        run_and_check(ifl, orc, S, T, X, Y, version)


@pytest.mark.parametrize("ds", ["small", "medium"])
def test_lvc_datasets_full(ifl, orc, ds):
    # P:402 datasets at full size and full numT (outer and the per-step auto)
    S, T, X, Y = gen.LVC_DATASETS[ds]
    for v in ("outer", "auto"):
        run_and_check(ifl, orc, S, T, X, Y, v, sample=[0, S // 2, S - 1])


def test_lvc_large_sampled(ifl, orc):
    # large dataset in the bench's launch configuration; the oracle
    # recomputes sampled outer indices s (systems are independent across s)
    S, T, X, Y = gen.LVC_DATASETS["large"]
    run_and_check(ifl, orc, S, T, X, Y, "outer", sample=[0, 131, S - 1])


def test_lvc_guard_and_notfit(ifl, orc):
    ifl.set_thresholds("lvc", 4, 0)
    try:
        assert run_and_check(ifl, orc, 4, 2, 8, 16, "auto").version == "outer"  # numS >= t0 (R1)
        assert run_and_check(ifl, orc, 3, 2, 8, 16, "auto").version == "auto"   # else: per-site G3
        assert ifl.select("lvc", 4, 8, 16).version == "outer"
        assert ifl.select("lvc", 4, 8, 600).version == "auto"                   # fit clause
        # numY > 512 does not fit V_OUTER: forced -> ENOTFIT, auto -> per-step path
        assert run_and_check(ifl, orc, 5, 2, 3, 600, "auto").version == "auto"
        (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(1, 2, 3, 600, "cuda")
        with pytest.raises(ifl.IflError) as e:
            ifl.lvc(xs, ys, (ax, bx, cx), (ay, by, cy), 2, version="outer")
        assert e.value.code == ifl.IFL_ENOTFIT
    finally:
        ifl.reset_thresholds()


def test_lvc_zero_steps_and_empty(ifl):
    (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(2, 3, 8, 16, "cuda")
    x0, y0 = xs.clone(), ys.clone()
    for v in ("outer", "auto", "flat"):
        ifl.lvc(xs, ys, (ax, bx, cx), (ay, by, cy), 0, version=v)
        assert torch.equal(xs, x0) and torch.equal(ys, y0)
    e = torch.empty(0, 8, 16, device="cuda")
    ifl.lvc(e, torch.empty(0, 16, 8, device="cuda"), (ax, bx, cx), (ay, by, cy), 3)


def test_lvc_tune_installs_t0(ifl):
    # the outermost guard's threshold from timing V_OUTER against the
    # per-step program on two training datasets
    try:
        t0, _, tbl = ifl.tune("lvc", [(16, 8, 32, 256), (4, 8, 256, 32)], reps=2, cost=1)
        assert np.isfinite(tbl[:, 0]).all() and np.isfinite(tbl[:, 2]).all() and np.isinf(tbl[:, 1]).all()
        assert ifl.get_thresholds("lvc")[0] == t0
    finally:
        ifl.reset_thresholds()


@pytest.mark.parametrize("version", ["outer", "middle", "flat"])
def test_lvc_step_by_step(ifl, orc, version):
    """The per-step bar behind the numT * 1e-5 loop bound (R13), checked
    directly: every step of the loop (one ifl_lvc step on the GPU's f32 state)
    is within the tridag bar 1e-5 * max(1, ||x||_inf) of the oracle's exact
    step from the same state -- the loop bound's only slack is the sum over
    steps, and the matrices' row margin keeps step errors from growing."""
    numS, numT, numX, numY = 2, 16, 32, 256
    (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(21, numS, numX, numY)
    xd, yd = xs.cuda(), ys.cuda()
    xc = tuple(t.cuda() for t in (ax, bx, cx))
    yc = tuple(t.cuda() for t in (ay, by, cy))
    co = [t.numpy() for t in (ax, bx, cx, ay, by, cy)]
    for step in range(numT):
        x0, y0 = xd.cpu().numpy().copy(), yd.cpu().numpy().copy()
        ifl.lvc(xd, yd, xc, yc, 1, version=version)
        want_x, want_y = orc.lvc(*co, x0, y0, 1)
        for got, want in ((xd.cpu().numpy(), want_x), (yd.cpu().numpy(), want_y)):
            err = np.abs(got.astype(np.float64) - want).max()
            assert err <= 1e-5 * max(1.0, np.abs(want).max()), f"{version} step {step}: {err:.3g}"
