"""GPU parity for tridag (batched tridiagonal solves via three scans,
P:400-420) against the oracle's Thomas algorithm in double.  Bound
(DESIGN.md): per system, max_j |x_j - x*_j| <= 1e-5 * max(1, ||x*||_inf)
on the diagonally dominant LocVolCalib-like systems of the input recipe."""
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


def check(orc, a, b, c, y, x, R):
    want = orc.tridag(a.numpy(), b.numpy(), c.numpy(), y.numpy(), R)
    got = x.cpu().numpy().astype(np.float64)
    scale = np.maximum(1.0, np.abs(want).max(axis=1, keepdims=True))
    err = np.abs(got - want) / scale
    assert err.max() <= 1e-5, f"max scaled err {err.max():.3g} at {np.unravel_index(err.argmax(), err.shape)}"


SHAPES = [(1, 1, 1), (3, 2, 1), (7, 5, 7), (512, 256, 32), (4096, 32, 256), (100, 1000, 10), (64, 33, 3),
          (5, 4096, 5), (2, 5000, 1)]


@pytest.mark.parametrize("version", ["top", "middle", "flat", "auto"])
def test_tridag_versions(ifl, orc, version):
    for (S, L, R) in SHAPES:
        if version == "middle" and L > 4096:
            continue
        a, b, c, y = gen.tridag_system(7, S, L, R)
        x = ifl.tridag(a.cuda(), b.cuda(), c.cuda(), y.cuda(), version=version)
        check(orc, a, b, c, y, x, R)


def test_tridag_middle_notfit(ifl):
    a, b, c, y = gen.tridag_system(7, 2, 5000, 1)
    with pytest.raises(ifl.IflError) as e:
        ifl.tridag(a.cuda(), b.cuda(), c.cuda(), y.cuda(), version="middle")
    assert e.value.code == ifl.IFL_ENOTFIT


def test_tridag_poisson_closed_form(ifl):
    # tridiag(-1, 2, -1) x = 1 -> x_j = (j+1)(L-j)/2
    for v in ("top", "middle", "flat"):
        for L in (1, 5, 32):
            a = torch.full((1, L), -1.0, device="cuda")
            b = torch.full((1, L), 2.0, device="cuda")
            c = torch.full((1, L), -1.0, device="cuda")
            y = torch.ones(3, L, device="cuda")
            x = ifl.tridag(a, b, c, y, version=v).cpu().numpy()
            j = np.arange(L)
            np.testing.assert_allclose(x, np.tile((j + 1) * (L - j) / 2.0, (3, 1)), rtol=2e-5, atol=1e-5)


@pytest.mark.parametrize("ds", ["small", "medium", "large"])
def test_config3_locvolcalib_sites(ifl, orc, ds):
    """BASELINE.json configs[3]: both tridag sites of one LocVolCalib time step
    (P:402 sizes): X-site S = numS*numX systems of L = numY, coefficients
    [numX][numY]; Y-site S = numS*numY of L = numX, coefficients [numY][numX].
    Sampled systems are checked (the large one has 65536 x 256)."""
    numS, numX, numY = {"small": (16, 32, 256), "medium": (128, 256, 32), "large": (256, 256, 256)}[ds]
    for (S, L, R) in ((numS * numX, numY, numX), (numS * numY, numX, numY)):
        a, b, c, y = gen.tridag_system(8, S, L, R)
        rows = sorted(set([0, 1, R - 1, R, S // 2, S - 1]))
        for v in ("top", "middle", "flat", "auto"):
            x = ifl.tridag(a.cuda(), b.cuda(), c.cuda(), y.cuda(), version=v)
            ys = y[rows]
            # the oracle solves only the sampled systems: their coefficient rows
            rr = [s % R for s in rows]
            want = orc.tridag(a[rr].numpy(), b[rr].numpy(), c[rr].numpy(), ys.numpy(), len(rr))
            # coefficient row of sampled system k is k % len(rr) == k: consistent
            got = x[rows].cpu().numpy().astype(np.float64)
            scale = np.maximum(1.0, np.abs(want).max(axis=1, keepdims=True))
            assert (np.abs(got - want) / scale).max() <= 1e-5, (ds, S, L, v)
