"""Pins for the CPU oracle (oracle/ifl_oracle.c) against things other than
itself: the paper's worked example, closed forms, brute force with
an independent formulation (Python ints / numpy / math.fsum), algebraic
invariants, and textbook/library routines (scipy banded solver).

A plausible mistake anywhere in the oracle -- a dropped term, an exclusive
instead of inclusive scan, a wrong index, a transposed operand, a missing
neutral element, non-wrapping overflow -- fails at least one test here.
"""
import functools
import math
import os

import numpy as np
import pytest
import torch

import ifl_inputs as gen

HERE = os.path.dirname(os.path.abspath(__file__))
INT_OPS = ["sum", "prod", "min", "max", "and", "or", "xor"]
F32_OPS = ["sum", "prod", "min", "max"]
MAPS = ["id", "sq", "abs"]


def load_golden():
    rows = {}
    for line in open(os.path.join(HERE, "golden", "p116_worked_example.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, val = (s.strip() for s in line.split("|"))
        rows[name] = np.array([[int(v) for v in r.split(",")] for r in val.split(";")])
    return rows


# ----------------------------------------------------------------- P:116


def test_p116_worked_example(orc):
    g = load_golden()
    x = g["input"].astype(np.int32)
    np.testing.assert_array_equal(orc.segscan(x, "sum", "id", 0), g["segscan_sum"])
    np.testing.assert_array_equal(orc.segred(x, "sum", "id", 0), g["segred_sum"][:, 0])
    xf = x.astype(np.float32)
    np.testing.assert_array_equal(orc.segscan(xf, "sum", "id", 0.0), g["segscan_sum"])
    np.testing.assert_array_equal(orc.segred(xf, "sum", "id", 0.0), g["segred_sum"][:, 0])


# ----------------------------------------------------- empty / neutral


@pytest.mark.parametrize("op", INT_OPS)
def test_empty_segment_is_neutral(orc, op):
    # reduce (+) 0 [] = 0 (empty list => the neutral element alone).
    x = np.zeros((5, 0), np.int32)
    np.testing.assert_array_equal(orc.segred(x, op, "id", 1234), np.full(5, 1234))
    assert orc.segscan(x, op).shape == (5, 0)
    if op in F32_OPS:
        xf = np.zeros((3, 0), np.float32)
        np.testing.assert_array_equal(orc.segred(xf, op, "id", 2.5), np.full(3, 2.5))


def test_neutral_element_applied_once(orc):
    # d (+) a1 (+) ... : with d = 7 and sum, the result is 7 + sum (not 7*m + sum).
    x = np.ones((2, 5), np.int32)
    np.testing.assert_array_equal(orc.segred(x, "sum", "id", 7), [12, 12])
    np.testing.assert_array_equal(orc.segscan(x, "sum", "id", 7), [[8, 9, 10, 11, 12]] * 2)


# ---------------------------------------------------------- closed forms


def test_closed_form_sum_0_to_k_config1(orc):
    n = m = 1024  # BASELINE.json configs[0]
    j = np.arange(m, dtype=np.int64)
    x = np.broadcast_to(j, (n, m)).astype(np.int32)
    np.testing.assert_array_equal(orc.segred(x, "sum"), np.full(n, m * (m - 1) // 2))
    i = np.arange(n, dtype=np.int64)[:, None]
    x2 = (i * m + j).astype(np.int32)
    want = m * m * np.arange(n, dtype=np.int64) + m * (m - 1) // 2
    assert want.max() < 2**31
    np.testing.assert_array_equal(orc.segred(x2, "sum"), want)


def test_closed_form_wraparound(orc):
    # sum of 0..k-1 with k = 2^17 exceeds 2^31: must wrap mod 2^32.
    k = 1 << 17
    x = np.arange(k, dtype=np.int64).astype(np.int32)[None, :]
    want = (k * (k - 1) // 2) % 2**32
    want = want - 2**32 if want >= 2**31 else want
    assert orc.segred(x, "sum")[0] == want
    # product of 2's: 2^40 mod 2^32 = 0
    assert orc.segred(np.full((1, 40), 2, np.int32), "prod")[0] == 0
    assert orc.segred(np.full((1, 31), 2, np.int32), "prod")[0] == -2**31


@pytest.mark.parametrize("m", [1, 7, 64, 1000])
def test_closed_form_scans(orc, m):
    ones = np.ones((3, m), np.int32)
    np.testing.assert_array_equal(orc.segscan(ones, "sum"), np.tile(np.arange(1, m + 1), (3, 1)))
    j = np.tile(np.arange(m, dtype=np.int32), (2, 1))
    np.testing.assert_array_equal(orc.segscan(j, "sum"), np.tile(np.arange(m) * (np.arange(m) + 1) // 2, (2, 1)))
    np.testing.assert_array_equal(orc.segscan(j, "max"), j)             # increasing row
    np.testing.assert_array_equal(orc.segscan(j[:, ::-1].copy(), "min"), j[:, ::-1])
    # reverse scan of ones: m - j
    np.testing.assert_array_equal(orc.segscan(ones, "sum", reverse=True), np.tile(np.arange(m, 0, -1), (3, 1)))
    jf = j.astype(np.float32)
    np.testing.assert_array_equal(orc.segscan(jf, "sum"), np.tile(np.arange(m) * (np.arange(m) + 1) / 2, (2, 1)))


def test_closed_form_min_max_permutation(orc):
    rng = np.random.default_rng(0)
    m = 513
    x = np.stack([rng.permutation(m) for _ in range(8)]).astype(np.int32)
    np.testing.assert_array_equal(orc.segred(x, "min"), np.zeros(8))
    np.testing.assert_array_equal(orc.segred(x, "max"), np.full(8, m - 1))
    np.testing.assert_array_equal(orc.segred(x.astype(np.float32) - 256, "min"), np.full(8, -256.0))


def test_maps(orc):
    x = np.array([[-3, 2, -2**31]], np.int32)
    assert orc.segred(x[:, :2], "sum", "sq")[0] == 13
    assert orc.segred(x[:, :2], "sum", "abs")[0] == 5
    assert orc.segred(x[:, 2:], "sum", "abs")[0] == -2**31  # |INT_MIN| wraps
    xf = np.array([[-1.5, 0.5]], np.float32)
    assert orc.segred(xf, "sum", "sq")[0] == 2.5
    assert orc.segred(xf, "max", "abs")[0] == 1.5


# ------------------------------------------- brute force, independent forms


def _ref_op(op):
    M = 1 << 32
    if op == "sum":
        return lambda a, b: (a + b) % M
    if op == "prod":
        return lambda a, b: (a * b) % M
    if op == "min":
        return lambda a, b: a if _s(a) <= _s(b) else b
    if op == "max":
        return lambda a, b: a if _s(a) >= _s(b) else b
    if op == "and":
        return lambda a, b: a & b
    if op == "or":
        return lambda a, b: a | b
    return lambda a, b: a ^ b


def _s(u):
    return u - (1 << 32) if u >= (1 << 31) else u


def _ref_map(f):
    M = 1 << 32
    return {"id": lambda v: v % M, "sq": lambda v: (v * v) % M, "abs": lambda v: abs(v) % M}[f]


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("op", INT_OPS)
def test_brute_force_int(orc, seed, op):
    """All (n, m) in [0..8]^2: the O(m) running oracle against an O(m^2)
    re-definition in Python ints (each scan element a fresh reduce)."""
    fn = _ref_op(op)
    d = int(gen.generate("I32_FULL", seed + 100, 1)[0])
    for f in MAPS:
        mp = _ref_map(f)
        for n in range(9):
            for m in range(9):
                x = gen.matrix("I32_SMALL" if op == "prod" else "I32_FULL", seed, n, m).numpy()
                red = orc.segred(x, op, f, d)
                scn = orc.segscan(x, op, f, d)
                for i in range(n):
                    row = [mp(int(v)) for v in x[i]]
                    want = functools.reduce(fn, row, d % (1 << 32))
                    assert red[i] == _s(want)
                    for j in range(m):
                        assert scn[i, j] == _s(functools.reduce(fn, row[: j + 1], d % (1 << 32)))


def test_against_numpy_int(orc):
    x = gen.matrix("I32_FULL", 1, 64, 300).numpy()
    s = (x.astype(np.int64).sum(1) % 2**32)
    s = np.where(s >= 2**31, s - 2**32, s)
    np.testing.assert_array_equal(orc.segred(x, "sum"), s)
    np.testing.assert_array_equal(orc.segred(x, "xor"), np.bitwise_xor.reduce(x, axis=1))
    np.testing.assert_array_equal(orc.segred(x, "and"), np.bitwise_and.reduce(x, axis=1))
    np.testing.assert_array_equal(orc.segred(x, "or"), np.bitwise_or.reduce(x, axis=1))
    np.testing.assert_array_equal(orc.segred(x, "min"), x.min(1))
    np.testing.assert_array_equal(orc.segred(x, "max"), x.max(1))
    c = np.cumsum(x.astype(np.int64), 1) % 2**32
    np.testing.assert_array_equal(orc.segscan(x, "sum"), np.where(c >= 2**31, c - 2**32, c))
    np.testing.assert_array_equal(orc.segscan(x, "max"), np.maximum.accumulate(x, 1))


@pytest.mark.parametrize("f", MAPS)
def test_f32_against_fsum(orc, f):
    """f32 sums: the double-accumulating oracle vs the exactly-rounded
    math.fsum of the same f32 terms; |err| <= m * 2^-53 * sum|f(x)|."""
    x = gen.matrix("F32_SIGNED", 2, 16, 4096).numpy()
    fx = {"id": x, "sq": (x * x).astype(np.float32), "abs": np.abs(x)}[f]
    out, ab = orc.segred(x, "sum", f, 0.0, with_absum=True)
    for i in range(x.shape[0]):
        exact = math.fsum(fx[i].astype(np.float64))
        assert abs(out[i] - exact) <= x.shape[1] * 2**-53 * ab[i]
        assert ab[i] == pytest.approx(np.abs(fx[i].astype(np.float64)).sum(), rel=1e-12)
    np.testing.assert_array_equal(orc.segred(x, "max", f), fx.max(1))
    np.testing.assert_array_equal(orc.segred(x, "min", f), fx.min(1))
    sc, sab = orc.segscan(x[:2, :300], "sum", f, 0.0, with_absum=True)
    np.testing.assert_allclose(sc, np.cumsum(fx[:2, :300].astype(np.float64), 1), rtol=0, atol=1e-9)
    np.testing.assert_allclose(sab, np.cumsum(np.abs(fx[:2, :300].astype(np.float64)), 1), rtol=1e-12)


def test_f32_prod_against_numpy(orc):
    x = (0.5 + gen.matrix("F32_UNIT", 9, 8, 50).numpy()).astype(np.float32)
    np.testing.assert_allclose(orc.segred(x, "prod"), np.prod(x.astype(np.float64), 1), rtol=1e-12)


def test_f32_exact_distribution_any_order(orc):
    """F32_EXACT: |partial sums| stay < 2^24, so every association is exact;
    the literal f32 left-to-right oracle equals the double one bit for bit."""
    x = gen.matrix("F32_EXACT", 3, 4, 1 << 20).numpy()
    pre = np.cumsum(x.astype(np.int64), 1)
    assert (pre.max(1) - np.minimum(pre.min(1), 0)).max() < 2**24
    np.testing.assert_array_equal(orc.segred_f32_literal(x), orc.segred(x).astype(np.float32))
    np.testing.assert_array_equal(orc.segred(x), x.astype(np.int64).sum(1))


# ------------------------------------------------------------ invariants


@pytest.mark.parametrize("op", INT_OPS)
def test_associativity_and_identity(orc, op):
    t = gen.matrix("I32_FULL", 11, 200, 3).numpy()
    whole = orc.segred(t, op)
    left = orc.segred(t[:, :2], op)
    two = np.stack([left, t[:, 2]], 1).astype(np.int32)
    np.testing.assert_array_equal(orc.segred(two, op), whole)             # (a+b)+c
    right = orc.segred(t[:, 1:], op)
    np.testing.assert_array_equal(orc.segred(np.stack([t[:, 0], right], 1).astype(np.int32), op), whole)
    # canonical d is neutral: d (+) x = x
    np.testing.assert_array_equal(orc.segred(t[:, :1], op), t[:, 0])


@pytest.mark.parametrize("op", INT_OPS)
def test_scan_last_column_and_split(orc, op):
    x = gen.matrix("I32_FULL", 12, 37, 129).numpy()
    np.testing.assert_array_equal(orc.segscan(x, op)[:, -1], orc.segred(x, op))
    for k in (0, 1, 64, 128, 129):  # split invariance (multi-GPU inner split relies on it)
        parts = np.stack([orc.segred(x[:, :k], op), orc.segred(x[:, k:], op)], 1).astype(np.int32)
        np.testing.assert_array_equal(orc.segred(parts, op), orc.segred(x, op))


def test_g4_column_identity(orc):
    # reduce (map (+)) (replicate m 0) M == map (reduce (+) 0) (transpose M)
    M = gen.matrix("I32_FULL", 13, 33, 70).numpy()
    np.testing.assert_array_equal(orc.colred(M), orc.segred(np.ascontiguousarray(M.T)))
    np.testing.assert_array_equal(orc.colred(M), (M.astype(np.int64).sum(0) + 2**31) % 2**32 - 2**31)
    Mf = gen.matrix("F32_EXACT", 13, 33, 70).numpy()
    np.testing.assert_array_equal(orc.colred(Mf), Mf.astype(np.float64).sum(0))


# --------------------------------------------------------------- redomap2


def _bf16_bits(t: torch.Tensor) -> np.ndarray:
    return t.contiguous().view(torch.int16).numpy().view(np.uint16)


def test_redomap2_closed_forms(orc):
    n, m, p = 5, 37, 6
    C = orc.redomap2(np.ones((n, m), np.float32), np.ones((p, m), np.float32))
    np.testing.assert_array_equal(C, np.full((n, p), m))
    # A = 1, B[k][j] = k mod 16 (B given as [m][p])  ->  C[i][j] = sum_k (k mod 16)
    B = np.tile((np.arange(m) % 16)[:, None], (1, p)).astype(np.float32)
    C = orc.redomap2(np.ones((n, m), np.float32), B, b_kmajor=False)
    np.testing.assert_array_equal(C, np.full((n, p), (np.arange(m) % 16).sum()))
    # A = I (n = m) -> C = B  (B as [m][p], and as transpose [p][m])
    Bm = gen.matrix("F32_SIGNED", 6, m, p).numpy()
    I = np.eye(m, dtype=np.float32)
    np.testing.assert_array_equal(orc.redomap2(I, Bm, b_kmajor=False), Bm)
    np.testing.assert_array_equal(orc.redomap2(I, np.ascontiguousarray(Bm.T), b_kmajor=True), Bm)


def test_redomap2_against_numpy(orc):
    A = gen.matrix("F32_SIGNED", 6, 17, 45).numpy()
    Bt = gen.matrix("F32_SIGNED", 7, 23, 45).numpy()
    C, ab = orc.redomap2(A, Bt, b_kmajor=True, with_abs=True)
    np.testing.assert_allclose(C, A.astype(np.float64) @ Bt.T.astype(np.float64), rtol=0, atol=1e-12)
    np.testing.assert_allclose(ab, np.abs(A.astype(np.float64)) @ np.abs(Bt.T.astype(np.float64)), rtol=1e-12)
    Ab = gen.matrix("BF16_SIGNED", 6, 9, 40)
    Bb = gen.matrix("BF16_SIGNED", 7, 40, 11)
    C = orc.redomap2(_bf16_bits(Ab), _bf16_bits(Bb), b_kmajor=False)
    np.testing.assert_allclose(C, Ab.double().numpy() @ Bb.double().numpy(), rtol=0, atol=1e-12)


# ----------------------------------------------------------------- tridag


def test_tridag_poisson_closed_form(orc):
    # tridiag(-1, 2, -1) x = 1  ->  x_j = (j+1)(L-j)/2  (j = 0..L-1)
    for L in (1, 2, 5, 32):
        a = np.full((1, L), -1, np.float32)
        b = np.full((1, L), 2, np.float32)
        c = np.full((1, L), -1, np.float32)
        y = np.ones((3, L), np.float32)
        x = orc.tridag(a, b, c, y, 1)
        j = np.arange(L)
        np.testing.assert_allclose(x, np.tile((j + 1) * (L - j) / 2.0, (3, 1)), rtol=1e-12)


def test_tridag_against_scipy_and_residual(orc):
    from scipy.linalg import solve_banded
    S, L, R = 12, 33, 4
    a, b, c, y = (t.numpy() for t in gen.tridag_system(7, S, L, R))
    x = orc.tridag(a, b, c, y, R)
    for s in range(S):
        r = s % R  # coefficient row shared every R systems
        ab = np.zeros((3, L))
        ab[0, 1:] = c[r, :-1]
        ab[1] = b[r]
        ab[2, :-1] = a[r, 1:]
        want = solve_banded((1, 1), ab, y[s].astype(np.float64))
        np.testing.assert_allclose(x[s], want, rtol=1e-10, atol=1e-12)
        Ax = b[r] * x[s]
        Ax[1:] += a[r, 1:] * x[s, :-1]
        Ax[:-1] += c[r, :-1] * x[s, 1:]
        assert np.abs(Ax - y[s]).max() < 1e-12


# ---- segscan_seeded (ifl_segscan_seeded): per-row d
def test_seeded_closed_form(orc):
    # ones with seed s_i: out[i, j] = s_i + j + 1
    n, m = 4, 9
    seed = np.array([0, 5, -3, 100], np.int32)
    got = orc.segscan_seeded(np.ones((n, m), np.int32), seed, "sum")
    np.testing.assert_array_equal(got, seed[:, None] + np.arange(1, m + 1)[None, :])
    # max with seed above every element: the row is constant seed
    x = np.arange(n * m, dtype=np.int32).reshape(n, m)
    np.testing.assert_array_equal(orc.segscan_seeded(x, np.full(n, 10**6, np.int32), "max"),
                                  np.full((n, m), 10**6, np.int32))


def test_seeded_continues_a_split_row(orc):
    # P:79 associativity: scanning columns [k, m) seeded with the inclusive
    # scan of [0, k) gives the tail of the full-row scan (the carry step of
    # the multi-GPU inner split)
    rng = np.random.default_rng(5)
    for op in ("sum", "min", "max", "xor"):
        x = rng.integers(-1000, 1000, size=(3, 40), dtype=np.int32)
        full = orc.segscan(x, op)
        for k in (1, 17, 39):
            tail = orc.segscan_seeded(np.ascontiguousarray(x[:, k:]), full[:, k - 1].copy(), op)
            np.testing.assert_array_equal(tail, full[:, k:])
    xf = rng.standard_normal((2, 50)).astype(np.float32)
    full = orc.segscan(xf, "sum")
    tail, ab = orc.segscan_seeded(np.ascontiguousarray(xf[:, 20:]), full[:, 19].astype(np.float32), "sum",
                                  with_absum=True)
    assert (np.abs(tail - full[:, 20:]) <= 1e-6 * (ab + 1)).all()


def test_seeded_equal_seeds_is_plain_scan(orc):
    x = np.arange(24, dtype=np.int32).reshape(3, 8)
    np.testing.assert_array_equal(orc.segscan_seeded(x, np.full(3, 7, np.int32), "sum"), orc.segscan(x, "sum", "id", 7))


# ------------------------------------------------------- lvc (Fig 6a loop)


def _spectral_powers(lam, L, T, y):
    """tridiag(-lam, 1+2 lam, -lam)^{-T} y by the sine eigenbasis of the
    Dirichlet second difference: v_k(j) = sin(pi k (j+1) / (L+1)),
    mu_k = 1 + 4 lam sin^2(pi k / (2 (L+1))) -- a closed form that shares
    nothing with the Thomas recurrence."""
    j = np.arange(L)
    k = np.arange(1, L + 1)
    V = np.sin(np.pi * np.outer(k, j + 1) / (L + 1))  # [k][j], V V^T = (L+1)/2 I
    mu = 1 + 4 * lam * np.sin(np.pi * k / (2 * (L + 1))) ** 2
    coef = (V @ y.T) * (2.0 / (L + 1)) * mu[:, None] ** (-T)
    return (V.T @ coef).T


def test_lvc_spectral_closed_form(orc):
    lam = 0.375  # exact in f32
    numS, numX, numY = 2, 5, 7
    for T in (0, 1, 3, 8):
        ax = np.full((numX, numY), -lam, np.float32)
        bx = np.full((numX, numY), 1 + 2 * lam, np.float32)
        ay = np.full((numY, numX), -lam, np.float32)
        by = np.full((numY, numX), 1 + 2 * lam, np.float32)
        (_, _, _), (_, _, _), xs, ys = gen.lvc_problem(3, numS, numX, numY)
        xs, ys = xs.numpy(), ys.numpy()
        xo, yo = orc.lvc(ax, bx, ax, ay, by, ay, xs, ys, T)
        want_x = _spectral_powers(lam, numY, T, xs.reshape(-1, numY).astype(np.float64)).reshape(xs.shape)
        want_y = _spectral_powers(lam, numX, T, ys.reshape(-1, numX).astype(np.float64)).reshape(ys.shape)
        np.testing.assert_allclose(xo, want_x, rtol=1e-11, atol=1e-12)
        np.testing.assert_allclose(yo, want_y, rtol=1e-11, atol=1e-12)


def _banded_matvec(a, b, c, x):
    """A x for A = tridiag(a[1:], b, c[:-1]) row by row (a[0], c[L-1] unused)."""
    Ax = b * x
    Ax[..., 1:] += a[..., 1:] * x[..., :-1]
    Ax[..., :-1] += c[..., :-1] * x[..., 1:]
    return Ax


def test_lvc_step_residuals_and_scipy(orc):
    # each step solves A x_t = x_{t-1} (residual by a plain matvec), and the
    # loop equals scipy's banded solver applied numT times
    from scipy.linalg import solve_banded
    numS, numX, numY, T = 3, 6, 9, 4
    (ax, bx, cx), (ay, by, cy), xs, ys = (v if isinstance(v, torch.Tensor) else tuple(t.numpy() for t in v)
                                          for v in gen.lvc_problem(5, numS, numX, numY))
    xs, ys = xs.numpy(), ys.numpy()
    prev_x, prev_y = xs.astype(np.float64), ys.astype(np.float64)
    for t in range(1, T + 1):
        xo, yo = orc.lvc(ax, bx, cx, ay, by, cy, xs, ys, t)
        rx = _banded_matvec(ax.astype(np.float64)[None], bx.astype(np.float64)[None], cx.astype(np.float64)[None], xo) - prev_x
        ry = _banded_matvec(ay.astype(np.float64)[None], by.astype(np.float64)[None], cy.astype(np.float64)[None], yo) - prev_y
        assert np.abs(rx).max() < 1e-12 and np.abs(ry).max() < 1e-12
        prev_x, prev_y = xo, yo
    # scipy, applied T times per system
    want = xs.astype(np.float64).copy()
    for s in range(numS):
        for x in range(numX):
            ab = np.zeros((3, numY))
            ab[0, 1:] = cx[x, :-1]
            ab[1] = bx[x]
            ab[2, :-1] = ax[x, 1:]
            for _ in range(T):
                want[s, x] = solve_banded((1, 1), ab, want[s, x])
    np.testing.assert_allclose(prev_x, want, rtol=1e-10, atol=1e-12)


def test_lvc_sites_independent_and_tridag_consistent(orc):
    numS, numX, numY = 2, 4, 8
    (ax, bx, cx), (ay, by, cy), xs, ys = gen.lvc_problem(11, numS, numX, numY)
    ax, bx, cx, ay, by, cy, xs, ys = (t.numpy() for t in (ax, bx, cx, ay, by, cy, xs, ys))
    xo, yo = orc.lvc(ax, bx, cx, ay, by, cy, xs, ys, 2)
    xo2, _ = orc.lvc(ax, bx, cx, ay, by, cy, xs, np.zeros_like(ys), 2)
    np.testing.assert_array_equal(xo, xo2)  # the y-site never touches xsss
    # one step = one tridag call per site with coefficient rows shared (R9)
    x1, y1 = orc.lvc(ax, bx, cx, ay, by, cy, xs, ys, 1)
    np.testing.assert_allclose(x1.reshape(-1, numY), orc.tridag(ax, bx, cx, xs.reshape(-1, numY), numX), rtol=1e-14)
    np.testing.assert_allclose(y1.reshape(-1, numX), orc.tridag(ay, by, cy, ys.reshape(-1, numX), numY), rtol=1e-14)
    # the diffusion-like recipe keeps the state O(1) over many steps (no underflow)
    xT, _ = orc.lvc(ax, bx, cx, ay, by, cy, np.ones_like(xs), ys, 256)
    assert 0.05 < np.abs(xT).max() <= 1.0 + 1e-12


# ------------------------------------------- colscan (G4 with scan, NEXT-3)


def test_colscan_closed_forms(orc):
    n, m = 9, 5
    np.testing.assert_array_equal(orc.colscan(np.ones((n, m), np.int32)), np.tile(np.arange(1, n + 1)[:, None], (1, m)))
    x = np.tile(np.arange(n, dtype=np.int32)[:, None], (1, m))
    i = np.arange(n)
    np.testing.assert_array_equal(orc.colscan(x), np.tile((i * (i + 1) // 2)[:, None], (1, m)))
    # max-scan down a column that increases: the column itself
    np.testing.assert_array_equal(orc.colscan(x, "max"), x)
    assert orc.colscan(np.zeros((0, 3), np.int32)).shape == (0, 3)


@pytest.mark.parametrize("op", INT_OPS)
def test_colscan_g4_identity_and_numpy(orc, op):
    # G4: the column scan is the row scan of the transpose; its last row is colred
    M = gen.matrix("I32_FULL", 21, 13, 29).numpy()
    cs = orc.colscan(M, op, "sq")
    np.testing.assert_array_equal(cs, orc.segscan(np.ascontiguousarray(M.T), op, "sq").T)
    np.testing.assert_array_equal(cs[-1], orc.colred(M, op, "sq"))
    if op == "sum":  # numpy: square mod 2^32 in int64, cumsum, then wrap
        sq = (M.astype(np.int64) * M.astype(np.int64)) % 2**32
        np.testing.assert_array_equal(cs, ((sq.cumsum(0) + 2**31) % 2**32 - 2**31).astype(np.int32))


def test_colscan_f32_numpy_and_exact(orc):
    Mf = gen.matrix("F32_EXACT", 23, 40, 17).numpy()
    np.testing.assert_array_equal(orc.colscan(Mf), Mf.astype(np.float64).cumsum(0))
    Mu = gen.matrix("F32_SIGNED", 24, 50, 7).numpy()
    out, ab = orc.colscan(Mu, "sum", "abs", with_absum=True)
    np.testing.assert_allclose(out, np.abs(Mu).astype(np.float64).cumsum(0), rtol=1e-13)
    np.testing.assert_allclose(ab, out, rtol=1e-13)  # f = abs: the bound scale equals the result
    np.testing.assert_array_equal(orc.colscan(Mu, "min")[-1], orc.colred(Mu, "min"))


# ------------------------------------------- irregular segments (NEXT-4)


def _wrap(v):
    return ((np.asarray(v, dtype=np.int64) + 2**31) % 2**32 - 2**31).astype(np.int32)


def test_irr_regular_descriptor_equals_rows(orc):
    # offsets i*m describe the regular [n][m] nest: same results as the row oracle
    for op in INT_OPS:
        x = gen.matrix("I32_FULL", 41, 9, 13).numpy()
        off = np.arange(10, dtype=np.int64) * 13
        np.testing.assert_array_equal(orc.seg_irr(x, off, False, op, "sq"), orc.segred(x, op, "sq"))
        np.testing.assert_array_equal(orc.seg_irr(x, off, True, op, "abs"), orc.segscan(x, op, "abs").reshape(-1))


def test_irr_closed_forms_and_empty(orc):
    lens = np.array([0, 3, 0, 0, 1, 7, 0], np.int64)
    off = np.r_[0, np.cumsum(lens)]
    ones = np.ones(off[-1], np.int32)
    np.testing.assert_array_equal(orc.seg_irr(ones, off, False), lens)        # sum of ones = length
    pos = np.concatenate([np.arange(1, L + 1) for L in lens])
    np.testing.assert_array_equal(orc.seg_irr(ones, off, True), pos)          # scan of ones = j + 1
    for op in INT_OPS:                                                        # empty reduce = d
        out = orc.seg_irr(ones, off, False, op, d=-5)
        assert (out[lens == 0] == -5).all()
    with pytest.raises(ValueError):
        orc.seg_irr(ones, np.array([0, 5, 3, 11], np.int64), False)           # decreasing descriptor


def test_irr_numpy_cumsum_and_brute_force(orc):
    rng = np.random.default_rng(3)
    for trial in range(5):
        lens = rng.integers(0, 9, size=rng.integers(1, 40)).astype(np.int64)
        off = np.r_[0, np.cumsum(lens)]
        x = gen.generate("I32_FULL", 50 + trial, int(off[-1])).numpy()
        cs = np.r_[0, np.cumsum(x.astype(np.int64))]
        np.testing.assert_array_equal(orc.seg_irr(x, off, False), _wrap(cs[off[1:]] - cs[off[:-1]]))
        seg_of = np.repeat(np.arange(len(lens)), lens)
        np.testing.assert_array_equal(orc.seg_irr(x, off, True), _wrap(cs[1:] - cs[off[:-1]][seg_of]))
        for op, fn in (("max", max), ("min", min), ("xor", lambda a, b: a ^ b)):
            want = []
            for i in range(len(lens)):  # brute force in Python ints
                acc = orc.canonical_ne(op, "i32")
                for k in range(off[i], off[i + 1]):
                    acc = fn(acc, int(x[k]))
                want.append(acc)
            np.testing.assert_array_equal(orc.seg_irr(x, off, False, op), np.array(want, np.int32))
        xf = gen.generate("F32_SIGNED", 60 + trial, int(off[-1])).numpy()
        got, ab = orc.seg_irr(xf, off, False, with_absum=True)
        want = np.array([math.fsum(xf[off[i]:off[i + 1]].astype(np.float64)) for i in range(len(lens))])
        assert (np.abs(got - want) <= 1e-12 * (ab + 1)).all()


def test_irr_f32_scan_against_numpy_and_fsum(orc):
    """oracle_segscan_irr_f32 (unpinned): per segment, the scan is
    d + numpy's float64 cumsum of f(x), its last element is math.fsum of the
    segment, min/max scans are numpy's accumulate, and absum restarts at every
    segment (a value carried across a boundary, or absum not reset, fails)."""
    rng = np.random.default_rng(5)
    for trial in range(6):
        lens = rng.integers(0, 12, size=rng.integers(1, 50)).astype(np.int64)
        lens[rng.integers(0, len(lens))] = 0                               # at least one empty segment
        off = np.r_[0, np.cumsum(lens)]
        xf = gen.generate("F32_SIGNED", 90 + trial, int(off[-1])).numpy()
        for f, fx in (("id", xf.astype(np.float64)), ("sq", (xf * xf).astype(np.float32).astype(np.float64)),
                      ("abs", np.abs(xf).astype(np.float64))):
            for d in (None, 1.5):
                dd = 0.0 if d is None else d
                got, ab = orc.seg_irr(xf, off, True, "sum", f, d, with_absum=True)
                for i in range(len(lens)):
                    a, b = off[i], off[i + 1]
                    if a == b:
                        continue
                    seg = fx[a:b]
                    np.testing.assert_allclose(got[a:b], dd + np.cumsum(seg), rtol=0, atol=1e-12 * (1 + np.abs(seg).sum()))
                    assert abs(got[b - 1] - math.fsum([dd] + list(seg))) <= 1e-12 * (1 + np.abs(seg).sum())
                    np.testing.assert_allclose(ab[a:b], np.cumsum(np.abs(seg)), rtol=1e-15, atol=0)
        for op, acc in (("min", np.minimum.accumulate), ("max", np.maximum.accumulate)):
            got = orc.seg_irr(xf, off, True, op)
            for i in range(len(lens)):
                a, b = off[i], off[i + 1]
                if a < b:
                    np.testing.assert_array_equal(got[a:b], acc(xf[a:b].astype(np.float64)))


def test_f32_reverse_scan(orc):
    """The reversed scan (tridag's back-substitution direction):
    out[i][j] = d (+) f(x[i][m-1]) (+) ... (+) f(x[i][j]) -- numpy's cumsum of the
    reversed row, reversed back; closed form m - j for ones; min/max by
    numpy's accumulate; absum is the reversed prefix of |f(x)|."""
    for (n, m) in [(1, 1), (3, 17), (5, 1000)]:
        ones = np.ones((n, m), np.float32)
        np.testing.assert_array_equal(orc.segscan(ones, "sum", reverse=True), np.tile(np.arange(m, 0, -1.0), (n, 1)))
        x = gen.matrix("F32_SIGNED", 33, n, m).numpy()
        got, ab = orc.segscan(x, "sum", "id", d=0.25, reverse=True, with_absum=True)
        want = 0.25 + np.cumsum(x[:, ::-1].astype(np.float64), axis=1)[:, ::-1]
        np.testing.assert_allclose(got, want, rtol=0, atol=1e-12 * (1 + np.abs(x).sum()))
        np.testing.assert_allclose(ab, np.cumsum(np.abs(x[:, ::-1]).astype(np.float64), axis=1)[:, ::-1], rtol=1e-14)
        for op, acc in (("min", np.minimum.accumulate), ("max", np.maximum.accumulate)):
            np.testing.assert_array_equal(orc.segscan(x, op, reverse=True),
                                          acc(x[:, ::-1].astype(np.float64), axis=1)[:, ::-1])
        xi = gen.matrix("I32_FULL", 34, n, m).numpy()
        np.testing.assert_array_equal(orc.segscan(xi, "sum", reverse=True),
                                      _wrap(np.cumsum(xi[:, ::-1].astype(np.int64), axis=1)[:, ::-1]))


# ------------------------------------------- segarg: tuple-valued (+) (NEXT-3)


def test_segarg_numpy_and_closed_forms(orc):
    x = gen.matrix("I32_SMALL", 51, 37, 53).numpy()  # many ties: values in [-1000, 1000]
    for which, npf in (("min", np.argmin), ("max", np.argmax)):
        val, idx = orc.segarg(x, which)
        np.testing.assert_array_equal(idx, npf(x, axis=1))                 # numpy: first occurrence
        np.testing.assert_array_equal(val, x[np.arange(37), idx])
        np.testing.assert_array_equal(val, orc.segred(x, which))           # the value half is segred
    xf = gen.matrix("F32_SIGNED", 52, 20, 31).numpy()
    v, i = orc.segarg(xf, "min")
    np.testing.assert_array_equal(i, np.argmin(xf, axis=1))
    # f32 argmax (unpinned): numpy's first occurrence, on data with
    # many ties (values rounded to 1/8) and on plain signed data
    xt = (np.round(gen.matrix("F32_SIGNED", 53, 40, 57).numpy() * 8) / 8).astype(np.float32)
    for xx in (xf, xt):
        for which, npf in (("max", np.argmax), ("min", np.argmin)):
            v, i = orc.segarg(xx, which)
            np.testing.assert_array_equal(i, npf(xx, axis=1))
            np.testing.assert_array_equal(v, xx[np.arange(xx.shape[0]), i])
    inc = np.tile(np.arange(9, dtype=np.float32), (3, 1))                  # increasing: argmax = last
    assert (orc.segarg(inc, "max")[1] == 8).all() and (orc.segarg(-inc, "max")[1] == 0).all()
    # closed forms: decreasing rows -> last index; constant rows -> index 0; empty rows -> (d, -1)
    dec = np.tile(np.arange(9, 0, -1, dtype=np.int32), (3, 1))
    assert (orc.segarg(dec, "min")[1] == 8).all() and (orc.segarg(dec, "max")[1] == 0).all()
    assert (orc.segarg(np.full((2, 5), 7, np.int32), "min")[1] == 0).all()
    big = np.full((2, 4), 2**31 - 1, np.int32)                             # equal to d: still index 0
    assert (orc.segarg(big, "min")[1] == 0).all()
    v, i = orc.segarg(np.zeros((3, 0), np.float32), "max")
    assert (i == -1).all() and np.isneginf(v).all()


# ---------------------------------------- segred2: nested reduce (G9 e_rec, NEXT-2)


def test_segred2_composition_and_closed_forms(orc):
    # the nest = the row oracle applied twice (inner over k, outer over m)
    x = gen.generate("I32_FULL", 71, 5 * 6 * 7).numpy().reshape(5, 6, 7)
    for op_o, op_i in (("sum", "max"), ("xor", "sum"), ("min", "and"), ("prod", "or")):
        inner = orc.segred(np.ascontiguousarray(x.reshape(30, 7)), op_i, "sq", 3).reshape(5, 6)
        want = orc.segred(np.ascontiguousarray(inner), op_o, "id", -2)
        np.testing.assert_array_equal(orc.segred2(x, op_o, op_i, "sq", -2, 3), want)
    # same operator at both levels = one flat reduce of each [m*k] row (associativity)
    np.testing.assert_array_equal(orc.segred2(x, "sum", "sum"), orc.segred(np.ascontiguousarray(x.reshape(5, 42)), "sum"))
    # closed form: x[i][j][q] = q -> sum over j of max over q = m*(k-1)
    q = np.tile(np.arange(7, dtype=np.int32), (4, 3, 1))
    np.testing.assert_array_equal(orc.segred2(q, "sum", "max"), np.full(4, 3 * 6))
    # empty levels: k = 0 -> every g = d_i; m = 0 -> d_o
    np.testing.assert_array_equal(orc.segred2(np.zeros((2, 3, 0), np.int32), "sum", "max", d_i=5), [15, 15])
    np.testing.assert_array_equal(orc.segred2(np.zeros((2, 0, 4), np.int32), "sum", "max", d_o=9), [9, 9])
    xf = gen.generate("F32_SIGNED", 72, 3 * 8 * 9).numpy().reshape(3, 8, 9)
    np.testing.assert_allclose(orc.segred2(xf, "sum", "max"), xf.astype(np.float64).max(axis=2).sum(axis=1), rtol=1e-12)
