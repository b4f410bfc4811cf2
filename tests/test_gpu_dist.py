"""GPU side of the device-level split (dist.py) on one B200: an NCCL
communicator of world size 1 (plumbing), and G "virtual shards" of one array
combined with the library's own kernels exactly as the inner split does
(SURVEY 4(3)(i)).  Checked against the oracle."""
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
    return m


def test_nccl_world1(ifl, orc):
    import torch.distributed as td
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        for op in ("sum", "max", "xor"):
            X = gen.matrix("I32_FULL", 8, 3, 100003)
            want = orc.segred(X.numpy(), op, "id", 5)
            for t_dev in (1, 2):
                plan = dist.plan_segred(3, 100003, 1, 0, t_dev)
                out = dist.segred_dist(X.cuda(), 3, 100003, op, "id", 5, plan=plan, gather=True)
                np.testing.assert_array_equal(out.cpu().numpy(), want)
    finally:
        td.destroy_process_group()


@pytest.mark.parametrize("G", [2, 4, 8])
def test_virtual_shards(ifl, orc, G):
    """Inner split on one GPU: column shards -> partials without d -> the
    library's segred over the [n][G] partial matrix -> d applied once."""
    n, m = 4, (1 << 20) + 3
    X = gen.matrix("I32_FULL", 8, n, m).cuda()
    for op in ("sum", "min", "xor", "prod"):
        Xo = X if op != "prod" else gen.matrix("I32_SMALL", 8, n, m).cuda()
        cuts = [(m * r) // G for r in range(G + 1)]
        parts = [ifl.segred(Xo[:, cuts[r]:cuts[r + 1]].contiguous(), op) for r in range(G)]
        stacked = torch.stack(parts, 1).contiguous()
        total = ifl.segred(stacked, op, ne=7)
        np.testing.assert_array_equal(total.cpu().numpy(), orc.segred(Xo.cpu().numpy(), op, "id", 7))


@pytest.mark.parametrize("G", [2, 8])
def test_virtual_shards_segscan(ifl, orc, G):
    """segscan inner split on one GPU, step by step as dist.segscan_dist runs
    it per rank: block totals without d -> carry-in d (+) lower totals ->
    seeded local scan; the concatenated blocks equal the full scan."""
    n, m = 3, (1 << 20) + 5
    for op in ("sum", "max", "xor"):
        X = gen.matrix("I32_FULL", 9, n, m).cuda()
        cuts = [(m * r) // G for r in range(G + 1)]
        blocks = [X[:, cuts[r]:cuts[r + 1]].contiguous() for r in range(G)]
        tots = torch.stack([ifl.segred(b, op) for b in blocks], 0)  # [G][n], what all_gather delivers
        outs = []
        for r in range(G):
            if r == 0:
                outs.append(ifl.segscan(blocks[0], op, ne=11))
            else:
                seed = ifl.segred(tots[:r].t().contiguous(), op, ne=11)
                outs.append(ifl.segscan(blocks[r], op, seed=seed))
        got = torch.cat(outs, 1).cpu().numpy()
        np.testing.assert_array_equal(got, orc.segscan(X.cpu().numpy(), op, "id", 11))


def test_nccl_world1_segscan(ifl, orc):
    import torch.distributed as td
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        X = gen.matrix("I32_FULL", 10, 2, 70001)
        for t_dev in (1, 2):
            plan = dist.plan_segred(2, 70001, 1, 0, t_dev)
            out = dist.segscan_dist(X.cuda(), 2, 70001, "sum", "id", 5, plan=plan)
            np.testing.assert_array_equal(out.cpu().numpy(), orc.segscan(X.numpy(), "sum", "id", 5))
    finally:
        td.destroy_process_group()


def test_redomap2_tridag_dist_gpu(ifl, orc):
    """redomap2_dist (outer and split-K plans, NCCL world 1) and tridag_dist
    with a block start that is not a multiple of R, on the GPU kernels."""
    import torch.distributed as td
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    td.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        n, m, p = 3, 4096, 40
        A = (gen.matrix("I32_SMALL", 11, n, m) % 5).float()
        Bt = (gen.matrix("I32_SMALL", 12, p, m) % 5).float()
        want = orc.redomap2(A.numpy(), Bt.numpy(), b_kmajor=True)
        for t_dev in (1, 4):
            plan = dist.plan_redomap2(n, m, p, 1, 0, t_dev)
            C = dist.redomap2_dist(A.cuda(), Bt.cuda(), n, m, p, plan=plan, gather=True)
            np.testing.assert_array_equal(C.cpu().numpy(), want)
    finally:
        td.destroy_process_group()
    S, L, R = 64, 256, 8
    a, b, c, y = gen.tridag_system(4, S, L, R)
    want = orc.tridag(a.numpy(), b.numpy(), c.numpy(), y.numpy(), R)
    lo = 11
    x = dist.tridag_dist(a.cuda(), b.cuda(), c.cuda(), y[lo:].contiguous().cuda(), lo).cpu().numpy()
    assert (np.abs(x - want[lo:]) <= 1e-5 * np.maximum(1.0, np.abs(want[lo:]).max(1, keepdims=True))).all()
