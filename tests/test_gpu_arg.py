"""GPU parity for the tuple-valued per-row argmin / argmax (ifl_segarg;
P:81-83) against the oracle: value AND index
bit-exact in every version (the operator resolves ties by index, so the
first occurrence is unique whatever the reduction order)."""
import numpy as np
import pytest
import torch

import ifl_inputs as gen

pytestmark = pytest.mark.gpu

VERS = ["top", "middle", "flat", "auto"]
SHAPES = [(1, 1), (3, 7), (100, 33), (5, 4095), (4, 4096), (2, 100003), (7, 1 << 17), (1000, 64), (1, 1 << 22),
          (3000, 4), (2001, 8), (999, 16), (700, 32)]


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
@pytest.mark.parametrize("which", ["min", "max"])
def test_segarg_versions(ifl, orc, version, which):
    for k, (n, m) in enumerate(SHAPES):
        for dist in ("I32_SMALL", "F32_SIGNED", "F32_EXACT"):  # I32_SMALL / F32_EXACT: many ties
            x = gen.matrix(dist, 60 + k, n, m)
            for mis in (False, True):
                if mis:
                    buf = torch.empty(n * m + 1, dtype=x.dtype, device="cuda")
                    xd = buf[1:].view(n, m)
                    xd.copy_(x)
                else:
                    xd = x.cuda()
                v, i = ifl.segarg(xd, which, version=version)
                wv, wi = orc.segarg(x.numpy(), which)
                np.testing.assert_array_equal(i.cpu().numpy(), wi)
                np.testing.assert_array_equal(v.cpu().numpy(), wv)


def test_segarg_edges(ifl):
    e = torch.empty(3, 0, dtype=torch.float32, device="cuda")
    v, i = ifl.segarg(e, "min")
    assert i.tolist() == [-1, -1, -1] and torch.isinf(v).all()
    x = torch.full((2, 9), 2**31 - 1, dtype=torch.int32, device="cuda")  # equal to d: first index
    for ver in VERS:
        assert ifl.segarg(x, "min", version=ver)[1].tolist() == [0, 0]
    # the value half equals segred min / max
    y = gen.matrix("I32_FULL", 70, 300, 500).cuda()
    for ver in VERS:
        assert torch.equal(ifl.segarg(y, "max", version=ver)[0], ifl.segred(y, "max"))
