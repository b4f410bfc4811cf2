"""Multi-process (world size 2, gloo, CPU) tests of the device-level split of
dist.py: plans, the single exchange step of the inner split, d applied once
after the collective, and the all-gather path used for bitwise operators.
The per-rank local segred is the CPU oracle here (tests may use it); on the
GPU box the same host logic calls the CUDA library."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as td
import torch.multiprocessing as mp

import ifl_inputs as gen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_local(x, op, f, ne):
    """Stands in for the GPU segred: same dtype in and out (f32 partials)."""
    import oracle
    xn = x.numpy()
    if xn.dtype == np.float64:
        xn = xn.astype(np.float32)
    r = oracle.segred(xn, op, f, ne)
    if r.dtype == np.float64:
        r = r.astype(np.float32)
    return torch.from_numpy(np.ascontiguousarray(r))


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    td.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    import oracle
    results = []
    try:
        cases = [("I32_FULL", op) for op in ("sum", "prod", "min", "max", "and", "or", "xor")] + \
                [("F32_EXACT", "sum"), ("F32_SIGNED", "max")]
        for (n, m) in [(1, 1000), (3, 77), (5, 2), (64, 31)]:
            for dist_name, op in cases:
                if op == "prod":
                    dist_name = "I32_SMALL"
                X = gen.matrix(dist_name, 5, n, m)
                d = 3 if X.dtype == torch.int32 else 1.5
                want = oracle.segred(X.numpy(), op, "id", d)
                for t_dev in (1, world + 1):  # force outer and inner
                    plan = dist.plan_segred(n, m, world, rank, t_dev)
                    blk = X[plan.lo:plan.hi] if plan.mode == "outer" else X[:, plan.lo:plan.hi].contiguous()
                    for gp in ((None, True) if plan.mode == "inner" else (None,)):
                        out = dist.segred_dist(blk, n, m, op, "id", d, plan=plan, gather=True,
                                               local_segred=_oracle_local, gather_partials=gp)
                        got = out.numpy()
                        if X.dtype == torch.int32:
                            ok = np.array_equal(got, want)
                        else:
                            ok = np.allclose(got, want, rtol=0, atol=1e-9)
                        results.append((plan.mode, n, m, dist_name, op, gp, bool(ok)))
        q.put((rank, results))
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, [("error", repr(e), False)]))
    finally:
        td.destroy_process_group()


def test_segred_dist_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, rows in res:
        bad = [r for r in rows if not r[-1]]
        assert not bad, f"rank {rank}: {bad[:5]}"
        assert any(r[0] == "outer" for r in rows) and any(r[0] == "inner" for r in rows)


def _oracle_local_scan(x, op, f, ne, seed):
    """Stands in for the GPU segscan (seeded when seed is given)."""
    import oracle
    xn = x.numpy()
    if seed is None:
        r = oracle.segscan(xn, op, f, ne)
    else:
        r = oracle.segscan_seeded(xn, seed.numpy(), op, f)
    if r.dtype == np.float64:
        r = r.astype(np.float32)
    return torch.from_numpy(np.ascontiguousarray(r))


def _scan_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    td.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    import oracle
    results = []
    try:
        cases = [("I32_FULL", op) for op in ("sum", "min", "max", "and", "or", "xor")] + \
                [("I32_SMALL", "prod"), ("F32_EXACT", "sum")]
        for (n, m) in [(1, 1000), (3, 77), (5, 2), (2, 1), (64, 31)]:
            for dist_name, op in cases:
                X = gen.matrix(dist_name, 6, n, m)
                d = 3 if X.dtype == torch.int32 else 1.5
                want = oracle.segscan(X.numpy(), op, "id", d)
                for t_dev in (1, world + 1):  # force outer and inner
                    plan = dist.plan_segred(n, m, world, rank, t_dev)
                    blk = X[plan.lo:plan.hi] if plan.mode == "outer" else X[:, plan.lo:plan.hi].contiguous()
                    out = dist.segscan_dist(blk, n, m, op, "id", d, plan=plan, local_segred=_oracle_local,
                                            local_segscan=_oracle_local_scan).numpy()
                    ref = want[plan.lo:plan.hi] if plan.mode == "outer" else want[:, plan.lo:plan.hi]
                    if X.dtype == torch.int32:
                        ok = np.array_equal(out, ref)
                    else:
                        ok = np.allclose(out, ref, rtol=0, atol=1e-9)
                    results.append((plan.mode, n, m, dist_name, op, bool(ok)))
        q.put((rank, results))
    except Exception as e:  # report instead of hanging the parent
        import traceback
        q.put((rank, [("error", traceback.format_exc(), False)]))
    finally:
        td.destroy_process_group()


def test_segscan_dist_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_scan_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, rows in res:
        bad = [r for r in rows if not r[-1]]
        assert not bad, f"rank {rank}: {bad[:5]}"
        assert any(r[0] == "outer" for r in rows) and any(r[0] == "inner" for r in rows)


def _mm_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    td.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    import oracle
    results = []

    def local_mm(A, B, b_kmajor):  # the oracle stands in for the GPU (fp64 -> fp32 partials)
        return torch.from_numpy(oracle.redomap2(A.numpy(), B.numpy(), b_kmajor=b_kmajor).astype(np.float32))

    def local_tri(a, b, c, y):
        return torch.from_numpy(oracle.tridag(a.numpy(), b.numpy(), c.numpy(), y.numpy(), a.shape[0])
                                .astype(np.float32))
    try:
        for (n, m, p) in [(1, 64, 1), (3, 50, 5), (8, 16, 3), (2, 1, 7)]:
            # small integers in f32: every partial and sum is exact
            A = (gen.matrix("I32_SMALL", 11, n, m) % 5).float()
            Bt = (gen.matrix("I32_SMALL", 12, p, m) % 5).float()
            want = oracle.redomap2(A.numpy(), Bt.numpy(), b_kmajor=True)
            for t_dev in (1, world + 1):
                for kmaj in (True, False):
                    plan = dist.plan_redomap2(n, m, p, world, rank, t_dev)
                    Bfull = Bt if kmaj else Bt.t().contiguous()
                    if plan.mode == "outer":
                        Ab, Bb = A[plan.lo:plan.hi].contiguous(), Bfull
                    else:
                        Ab = A[:, plan.lo:plan.hi].contiguous()
                        Bb = Bt[:, plan.lo:plan.hi].contiguous() if kmaj else Bfull[plan.lo:plan.hi].contiguous()
                    C = dist.redomap2_dist(Ab, Bb, n, m, p, plan=plan, b_kmajor=kmaj, gather=True,
                                           local_redomap2=local_mm).numpy()
                    results.append(("mm", plan.mode, n, m, p, kmaj, bool(np.array_equal(C, want))))
        # tridag: system split with a block start that is not a multiple of R
        S, L, R = 10, 16, 4
        a, b, c, y = gen.tridag_system(3, S, L, R)
        want = oracle.tridag(a.numpy(), b.numpy(), c.numpy(), y.numpy(), R)
        lo, hi = [(0, 5), (5, 10)][rank]
        x = dist.tridag_dist(a, b, c, y[lo:hi].contiguous(), lo, local_tridag=local_tri).numpy()
        results.append(("tridag", lo, hi, bool(np.allclose(x, want[lo:hi], rtol=1e-5, atol=1e-5))))
        q.put((rank, results))
    except Exception:
        import traceback
        q.put((rank, [("error", traceback.format_exc(), False)]))
    finally:
        td.destroy_process_group()


def test_redomap2_tridag_dist_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_mm_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, rows in res:
        bad = [r for r in rows if not r[-1]]
        assert not bad, f"rank {rank}: {bad[:5]}"
        assert any(r[:2] == ("mm", "outer") for r in rows) and any(r[:2] == ("mm", "inner") for r in rows)


def test_plans_cover_exactly():
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    for world in (1, 2, 3, 8):
        for (n, m) in [(1, 10), (7, 3), (100, 1), (8, 8)]:
            plans = [dist.plan_segred(n, m, world, r) for r in range(world)]
            assert len({p.mode for p in plans}) == 1
            if plans[0].mode == "outer":
                cover = [i for p in plans for i in range(p.lo, p.hi)]
                assert cover == list(range(n))
            else:
                cover = [j for p in plans for j in range(p.lo, p.hi)]
                assert cover == list(range(m))


# ------------------------------------------- colred / lvc / irregular splits


def _worker_ext(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    td.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ppopp_henriksenteo19_b200 import dist
    import oracle
    res = []
    try:
        def loc_col(x, op, f, ne):
            r = oracle.colred(x.numpy(), op, f, ne)
            return torch.from_numpy(np.ascontiguousarray(r.astype(x.numpy().dtype)))
        for (n, m) in [(7, 1), (5, 13), (64, 3), (2, 40)]:
            for op in ("sum", "min", "xor"):
                X = gen.matrix("I32_FULL", 9, n, m)
                want = oracle.colred(X.numpy(), op, "id", 5)
                for t_dev in (1, 10**9):  # force column split / row split
                    plan = dist.plan_colred(n, m, world, rank, t_dev)
                    blk = X[:, plan.lo:plan.hi].contiguous() if plan.mode == "outer" else X[plan.lo:plan.hi]
                    out = dist.colred_dist(blk, n, m, op, "id", 5, plan=plan, gather=True, local_colred=loc_col)
                    res.append(("colred", plan.mode, n, m, op, bool(np.array_equal(out.numpy(), want))))
        # lvc: numS split, each rank's block equals the oracle's rows of the full run
        xc, yc, xs, ys = gen.lvc_problem(3, 5, 4, 6)
        wx, wy = oracle.lvc(*(t.numpy() for t in xc + yc), xs.numpy(), ys.numpy(), 3)
        lo, hi = dist.rows_of(5, world, rank)

        def loc_lvc(xb, yb, xcf, ycf, T):
            gx, gy = oracle.lvc(*(t.numpy() for t in xcf + ycf), xb.numpy(), yb.numpy(), T)
            xb.copy_(torch.from_numpy(gx.astype(np.float32)))
            yb.copy_(torch.from_numpy(gy.astype(np.float32)))
        xb, yb = xs[lo:hi].clone(), ys[lo:hi].clone()
        dist.lvc_dist(xb, yb, xc, yc, 3, local_lvc=loc_lvc)
        res.append(("lvc", lo, hi, bool(np.allclose(xb.numpy(), wx[lo:hi], atol=1e-6) and
                                         np.allclose(yb.numpy(), wy[lo:hi], atol=1e-6))))
        # irregular: element-balanced segment ranges; concatenated per-rank results = the whole
        off = gen.irregular_offsets(4, 300, 10.0)
        x = gen.generate("I32_FULL", 8, int(off[-1]))
        want = oracle.seg_irr(x.numpy(), off, False, "sum")
        s0, s1 = dist.plan_irr(off, world, rank)

        def loc_irr(xb, o, op, f, ne):
            return torch.from_numpy(oracle.seg_irr(xb.numpy(), o.numpy(), False, op, f, ne))
        got = dist.segred_irr_dist(x, off, s0, s1, local=loc_irr)
        parts = [None] * world
        td.all_gather_object(parts, (s0, s1, got))
        whole = torch.cat([p[2] for p in sorted(parts, key=lambda p: p[0])]).numpy()
        cover = sorted((p[0], p[1]) for p in parts)
        res.append(("irr", s0, s1, bool(np.array_equal(whole, want) and cover[0][0] == 0 and cover[-1][1] == 300)))
        q.put((rank, res))
    except Exception as e:
        q.put((rank, [("error", repr(e), False)]))
    finally:
        td.destroy_process_group()


def test_colred_lvc_irr_dist_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_ext, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, res in out:
        bad = [r for r in res if not r[-1]]
        assert not bad, (rank, bad[:5])
        assert len(res) > 20


def _bench_worker(rank, world, port, q):
    """bench.py's N > 1 step (the weak-scaled sweep through dist.py), gloo on
    CPU with the oracle standing in for the GPU library: every rank's results
    equal the oracle on the global [2^k][world * 2^L / 2^k] arrays."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    td.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    import oracle
    results = []

    def local_scan(x, op, f, ne, seed):
        xn = x.numpy()
        if seed is not None:
            return torch.from_numpy(oracle.segscan_seeded(xn, seed.numpy(), op, f).astype(xn.dtype))
        return torch.from_numpy(np.ascontiguousarray(oracle.segscan(xn, op, f, ne).astype(xn.dtype)))
    try:
        L = 6
        shapes = bench.sharded_shapes(world, rank, log2n=L)
        # the global array of every shape: world blocks of 2^L int32, rank r's block at r * 2^L
        G = gen.generate("I32_FULL", 17, world << L)
        mine = G[rank << L:(rank + 1) << L].contiguous()
        outs = bench.sharded_step(mine, shapes, local_segred=_oracle_local, local_segscan=local_scan)
        for i, (ng, mg, plan, (nl, ml)) in enumerate(shapes):
            # rank r's block: rows [lo, hi) (outer) or columns [lo, hi) of every row (inner) of the global array
            blocks = []
            for r in range(world):
                p = __import__("paper_conf_ppopp_henriksenteo19_b200.dist", fromlist=["x"]).plan_segred(ng, mg, world, r)
                blocks.append((p, G[r << L:(r + 1) << L]))
            X = np.zeros((ng, mg), np.int32)
            for p, b in blocks:
                if p.mode == "outer":
                    X[p.lo:p.hi] = b.numpy().reshape(p.hi - p.lo, mg)
                else:
                    X[:, p.lo:p.hi] = b.numpy().reshape(ng, p.hi - p.lo)
            red, scan = outs[2 * i].numpy(), outs[2 * i + 1].numpy()
            want_red, want_scan = oracle.segred(X, "sum"), oracle.segscan(X, "sum")
            if plan.mode == "outer":
                ok = np.array_equal(red, want_red[plan.lo:plan.hi]) and np.array_equal(
                    scan, want_scan[plan.lo:plan.hi])
            else:
                ok = np.array_equal(red, want_red) and np.array_equal(scan, want_scan[:, plan.lo:plan.hi])
            results.append((plan.mode, ng, mg, bool(ok)))
        q.put((rank, results))
    except Exception:
        import traceback
        q.put((rank, [("error", traceback.format_exc(), False)]))
    finally:
        td.destroy_process_group()


def test_bench_sharded_step_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, rows in res:
        bad = [r for r in rows if not r[-1]]
        assert not bad, f"rank {rank}: {bad[:5]}"
        assert any(r[0] == "outer" for r in rows) and any(r[0] == "inner" for r in rows)
