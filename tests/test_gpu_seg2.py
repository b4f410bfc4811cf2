"""GPU parity for the nested reduce ifl_segred2 (G9's e_rec, P:311-332;
SURVEY 8(f) NEXT-2) against the oracle's triple loop: int32 and f32 min/max
bit-exact, f32 sums within 1e-5 * sum |f(x)| (+ |d|)."""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "flat", "auto"]
SHAPES = [(1, 1, 1), (3, 5, 7), (64, 33, 40), (7, 300, 5), (2, 17, 4100), (500, 8, 8), (1, 1000, 1000), (5, 0, 3),
          (4, 3, 0)]


@pytest.fixture(scope="module")
def ifl():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_henriksenteo19_b200 import build
    build.build()
    import paper_conf_ppopp_henriksenteo19_b200 as m
    m.reset_thresholds()
    return m


@pytest.mark.parametrize("version", VERS)
def test_segred2_versions(ifl, orc, version):
    for s, (n, m, k) in enumerate(SHAPES):
        xi = gen.generate("I32_FULL", 80 + s, n * m * k).view(n, m, k)
        for op_o, op_i, f in (("sum", "max", "id"), ("xor", "sum", "sq"), ("min", "and", "abs"), ("prod", "or", "id")):
            got = ifl.segred2(xi.cuda(), op_o, op_i, f, ne_o=3, ne_i=-7, version=version).cpu().numpy()
            np.testing.assert_array_equal(got, orc.segred2(xi.numpy(), op_o, op_i, f, 3, -7))
        xf = gen.generate("F32_SIGNED", 90 + s, n * m * k).view(n, m, k)
        got = ifl.segred2(xf.cuda(), "max", "min", version=version).cpu().numpy()
        np.testing.assert_array_equal(got, orc.segred2(xf.numpy(), "max", "min").astype(np.float32))
        got = ifl.segred2(xf.cuda(), "sum", "max", version=version).cpu().numpy().astype(np.float64)
        want = orc.segred2(xf.numpy(), "sum", "max")
        bound = 1e-5 * (np.abs(xf.numpy()).max(axis=2).sum(axis=1) if m * k else 0) + 1e-6
        fin = np.isfinite(want)  # k == 0: every inner max is -inf, so is the sum
        assert (got[~fin] == want[~fin]).all(), (version, n, m, k)
        assert (np.abs(got[fin] - want[fin]) <= np.broadcast_to(bound, want.shape)[fin]).all(), (version, n, m, k)


def test_segred2_equals_two_segreds(ifl):
    x = gen.generate("I32_FULL", 95, 300 * 40 * 70).view(300, 40, 70).cuda()
    inner = ifl.segred(x.view(-1, 70), "max")
    want = ifl.segred(inner.view(300, 40), "xor")
    for v in VERS:
        assert torch.equal(ifl.segred2(x, "xor", "max", version=v), want)
