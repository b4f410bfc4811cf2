"""CPU oracle for the incremental-flattening hot path -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ppopp_henriksenteo19_b200``) never does, and the
two share no code: this wrapper loads ``libifl_oracle.so`` built from
``oracle/ifl_oracle.c`` (plain C, -O2, no fast-math, single thread).

Every function cites the PAPER.md passage it follows (``P:<line>``, the
line of /root/reference/PAPER.md).  Pins live in ``tests/test_oracle.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ifl_oracle.c")
_LIB = os.path.join(_HERE, "libifl_oracle.so")

OPS = {"sum": 0, "prod": 1, "min": 2, "max": 3, "and": 4, "or": 5, "xor": 6}
MAPS = {"id": 0, "sq": 1, "abs": 2}

_c_i64 = ctypes.c_int64
_c_int = ctypes.c_int
_vp = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile libifl_oracle.so with gcc (plain C, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fno-fast-math",
             "-ffp-contract=off", "-o", _LIB, _SRC, "-lm"])
    return _LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        for name, argt in {
            "oracle_segred_i32": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_int32],
            "oracle_segscan_i32": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_int32, _c_int],
            "oracle_colred_i32": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_int32],
            "oracle_segred_f32": [_vp, _vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_double],
            "oracle_segscan_f32": [_vp, _vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_double, _c_int],
            "oracle_colred_f32": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_double],
            "oracle_colscan_i32": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_int32],
            "oracle_colscan_f32": [_vp, _vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_double],
            "oracle_segred_f32_literal": [_vp, _vp, _c_i64, _c_i64, _c_int, _c_int, ctypes.c_float],
            "oracle_redomap2": [_vp, _vp, _vp, _vp, _c_i64, _c_i64, _c_i64, _c_int, _c_int],
            "oracle_tridag": [_vp, _vp, _vp, _vp, _vp, _c_i64, _c_i64, _c_i64, _vp],
            "oracle_lvc": [_vp] * 10 + [_c_i64] * 4 + [_vp],
            "oracle_segred2_i32": [_vp, _vp, _c_i64, _c_i64, _c_i64, _c_int, _c_int, _c_int, ctypes.c_int32,
                                   ctypes.c_int32],
            "oracle_segred2_f32": [_vp, _vp, _c_i64, _c_i64, _c_i64, _c_int, _c_int, _c_int, ctypes.c_double,
                                   ctypes.c_double],
            "oracle_segarg_i32": [_vp, _vp, _vp, _c_i64, _c_i64, _c_int],
            "oracle_segarg_f32": [_vp, _vp, _vp, _c_i64, _c_i64, _c_int],
            "oracle_segred_irr_i32": [_vp, _vp, _vp, _c_i64, _c_int, _c_int, ctypes.c_int32],
            "oracle_segscan_irr_i32": [_vp, _vp, _vp, _c_i64, _c_int, _c_int, ctypes.c_int32],
            "oracle_segred_irr_f32": [_vp, _vp, _vp, _vp, _c_i64, _c_int, _c_int, ctypes.c_double],
            "oracle_segscan_irr_f32": [_vp, _vp, _vp, _vp, _c_i64, _c_int, _c_int, ctypes.c_double],
        }.items():
            fn = getattr(L, name)
            fn.argtypes = argt
            fn.restype = _c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(_vp)


def _i32(v) -> int:
    """Wrap a Python int to the int32 range (two's complement)."""
    return ((int(v) + 2**31) % 2**32) - 2**31


def _check(rc: int):
    if rc != 0:
        raise ValueError(f"oracle returned {rc}")


# Canonical neutral elements 0_(+) (reading C6a).
def canonical_ne(op: str, dtype: str):
    if dtype == "i32":
        return {"sum": 0, "prod": 1, "min": 2**31 - 1, "max": -2**31,
                "and": -1, "or": 0, "xor": 0}[op]
    return {"sum": 0.0, "prod": 1.0, "min": float("inf"), "max": float("-inf")}[op]


def segred(x: np.ndarray, op: str = "sum", f: str = "id", d=None, with_absum=False):
    """P:79/P:85/P:109: out[i] = d (+) f(x[i,0]) (+) ... (+) f(x[i,m-1]).

    int32 -> int32 (wrapping); float32 -> float64 (exact-ish reference)."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    if x.dtype == np.int32:
        d = canonical_ne(op, "i32") if d is None else int(d)
        out = np.empty(n, np.int32)
        _check(lib().oracle_segred_i32(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f],
                                       _i32(d)))
        return (out, None) if with_absum else out
    if x.dtype == np.float32:
        d = canonical_ne(op, "f32") if d is None else float(np.float32(d))
        out = np.empty(n, np.float64)
        ab = np.empty(n, np.float64)
        _check(lib().oracle_segred_f32(_ptr(x), _ptr(out), _ptr(ab), n, m, OPS[op], MAPS[f], d))
        return (out, ab) if with_absum else out
    raise TypeError(x.dtype)


def segscan(x: np.ndarray, op: str = "sum", f: str = "id", d=None, reverse=False, with_absum=False):
    """P:79 (inclusive, pinned by P:116) / P:113: per-row scanomap."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    if x.dtype == np.int32:
        d = canonical_ne(op, "i32") if d is None else int(d)
        out = np.empty((n, m), np.int32)
        _check(lib().oracle_segscan_i32(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f],
                                        _i32(d), int(reverse)))
        return (out, None) if with_absum else out
    if x.dtype == np.float32:
        d = canonical_ne(op, "f32") if d is None else float(np.float32(d))
        out = np.empty((n, m), np.float64)
        ab = np.empty((n, m), np.float64)
        _check(lib().oracle_segscan_f32(_ptr(x), _ptr(out), _ptr(ab), n, m, OPS[op], MAPS[f],
                                        d, int(reverse)))
        return (out, ab) if with_absum else out
    raise TypeError(x.dtype)


def segscan_seeded(x: np.ndarray, seed: np.ndarray, op: str = "sum", f: str = "id", with_absum=False):
    """P:79's scan with d replaced row by row (ifl_segscan_seeded):
    out[i,j] = seed[i] (+) f(x[i,0]) (+) ... (+) f(x[i,j]).  Row i is exactly
    segscan(x[i:i+1], d=seed[i]); for f32 the tolerance base adds |seed[i]|."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    outs, abs_ = [], []
    for i in range(n):
        o, ab = segscan(x[i:i + 1], op, f, d=seed[i], with_absum=True)
        outs.append(o)
        if ab is not None:
            abs_.append(ab + abs(float(seed[i])))
    out = np.concatenate(outs) if n else (np.empty((0, m), np.int32 if x.dtype == np.int32 else np.float64))
    if not with_absum:
        return out
    return out, (np.concatenate(abs_) if abs_ else None)


def colred(x: np.ndarray, op: str = "sum", f: str = "id", d=None):
    """P:156 (G4 left-hand side): column reduction of an [n][m] matrix."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    if x.dtype == np.int32:
        d = canonical_ne(op, "i32") if d is None else int(d)
        out = np.empty(m, np.int32)
        _check(lib().oracle_colred_i32(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f],
                                       _i32(d)))
        return out
    d = canonical_ne(op, "f32") if d is None else float(np.float32(d))
    out = np.empty(m, np.float64)
    _check(lib().oracle_colred_f32(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f], d))
    return out


def colscan(x: np.ndarray, op: str = "sum", f: str = "id", d=None, with_absum=False):
    """G4 with scan: out[i][j] = d (+) f(x[0][j]) (+) ... (+) f(x[i][j])."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    if x.dtype == np.int32:
        d = canonical_ne(op, "i32") if d is None else int(d)
        out = np.empty((n, m), np.int32)
        _check(lib().oracle_colscan_i32(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f], _i32(d)))
        return out
    d = canonical_ne(op, "f32") if d is None else float(np.float32(d))
    out = np.empty((n, m), np.float64)
    ab = np.empty((n, m), np.float64)
    _check(lib().oracle_colscan_f32(_ptr(x), _ptr(out), _ptr(ab), n, m, OPS[op], MAPS[f], d))
    return (out, ab) if with_absum else out


def segred_f32_literal(x: np.ndarray, op: str = "sum", f: str = "id", d=None):
    """Information only: P:79 left-to-right in f32 (not a parity reference)."""
    x = np.ascontiguousarray(x, dtype=np.float32)
    n, m = x.shape
    d = canonical_ne(op, "f32") if d is None else float(d)
    out = np.empty(n, np.float32)
    _check(lib().oracle_segred_f32_literal(_ptr(x), _ptr(out), n, m, OPS[op], MAPS[f], d))
    return out


def redomap2(A: np.ndarray, B: np.ndarray, b_kmajor: bool = True, with_abs=False):
    """C = xss x yss with B given as transpose yss ([p][m], b_kmajor)
    or as yss ([m][p]).  A/B float32, or uint16 holding bf16 bits."""
    A = np.ascontiguousarray(A)
    B = np.ascontiguousarray(B)
    n, m = A.shape
    p = B.shape[0] if b_kmajor else B.shape[1]
    assert (B.shape[1] if b_kmajor else B.shape[0]) == m
    in_dt = 0 if A.dtype == np.float32 else 1
    assert A.dtype == B.dtype and A.dtype in (np.float32, np.uint16)
    C = np.empty((n, p), np.float64)
    ab = np.empty((n, p), np.float64)
    _check(lib().oracle_redomap2(_ptr(A), _ptr(B), _ptr(C), _ptr(ab), n, m, p, in_dt, int(b_kmajor)))
    return (C, ab) if with_abs else C


def tridag(a, b, c, y, coef_rows: int):
    """Thomas algorithm in double (textbook; reading R8)."""
    a, b, c, y = (np.ascontiguousarray(v, dtype=np.float32) for v in (a, b, c, y))
    S, L = y.shape
    assert a.shape == b.shape == c.shape == (coef_rows, L)
    x = np.empty((S, L), np.float64)
    work = np.empty(max(L, 1), np.float64)
    rc = lib().oracle_tridag(_ptr(a), _ptr(b), _ptr(c), _ptr(y), _ptr(x), S, L, coef_rows, _ptr(work))
    _check(rc)
    return x


def lvc(ax, bx, cx, ay, by, cy, xsss, ysss, numT: int):
    """The LocVolCalib loop of Fig 6a: numT steps of
    ``map tridag`` over xsss [numS][numX][numY] (coefficients [numX][numY])
    and ysss [numS][numY][numX] (coefficients [numY][numX]); Thomas solves in
    double, state kept in double.  Returns (xsss', ysss') as float64."""
    ax, bx, cx, ay, by, cy, xsss, ysss = (np.ascontiguousarray(v, dtype=np.float32)
                                          for v in (ax, bx, cx, ay, by, cy, xsss, ysss))
    numS, numX, numY = xsss.shape
    assert ysss.shape == (numS, numY, numX)
    assert ax.shape == bx.shape == cx.shape == (numX, numY)
    assert ay.shape == by.shape == cy.shape == (numY, numX)
    xo = np.empty(xsss.shape, np.float64)
    yo = np.empty(ysss.shape, np.float64)
    work = np.empty(max(numX, numY, 1), np.float64)
    _check(lib().oracle_lvc(_ptr(ax), _ptr(bx), _ptr(cx), _ptr(ay), _ptr(by), _ptr(cy), _ptr(xsss), _ptr(ysss),
                            _ptr(xo), _ptr(yo), numS, int(numT), numX, numY, _ptr(work)))
    return xo, yo


def seg_irr(x: np.ndarray, offsets: np.ndarray, scan: bool, op: str = "sum", f: str = "id", d=None,
            with_absum=False):
    """Irregular segments (P:532 future work): segment i is
    x[offsets[i]:offsets[i+1]]; reduce (out [n]) or inclusive scan (out like x)
    of every segment as P:79 defines them; an empty segment reduces to d."""
    x = np.ascontiguousarray(x).reshape(-1)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    n = off.shape[0] - 1
    assert off[-1] == x.shape[0]
    if x.dtype == np.int32:
        d = canonical_ne(op, "i32") if d is None else int(d)
        out = np.empty(x.shape[0] if scan else n, np.int32)
        fn = lib().oracle_segscan_irr_i32 if scan else lib().oracle_segred_irr_i32
        _check(fn(_ptr(x), _ptr(out), _ptr(off), n, OPS[op], MAPS[f], _i32(d)))
        return (out, None) if with_absum else out
    d = canonical_ne(op, "f32") if d is None else float(np.float32(d))
    out = np.empty(x.shape[0] if scan else n, np.float64)
    ab = np.empty_like(out)
    fn = lib().oracle_segscan_irr_f32 if scan else lib().oracle_segred_irr_f32
    _check(fn(_ptr(x), _ptr(out), _ptr(ab), _ptr(off), n, OPS[op], MAPS[f], d))
    return (out, ab) if with_absum else out


def segarg(x: np.ndarray, which: str = "min"):
    """Tuple-valued reduction (argmin of NN): per row the
    (value, index) of the first minimum / maximum; m == 0 -> (d, -1)."""
    x = np.ascontiguousarray(x)
    n, m = x.shape
    val = np.empty(n, x.dtype)
    idx = np.empty(n, np.int32)
    fn = lib().oracle_segarg_i32 if x.dtype == np.int32 else lib().oracle_segarg_f32
    _check(fn(_ptr(x), _ptr(val), _ptr(idx), n, m, 1 if which == "max" else 0))
    return val, idx


def segred2(x: np.ndarray, op_o: str = "sum", op_i: str = "max", f: str = "id", d_o=None, d_i=None):
    """Nested reduce (G9's e_rec): out[i] = d_o (+)_j (d_i (x)_q f(x[i,j,q]))
    over an [n][m][k] array; (+) = op_o, (x) = op_i."""
    x = np.ascontiguousarray(x)
    n, m, k = x.shape
    if x.dtype == np.int32:
        do = canonical_ne(op_o, "i32") if d_o is None else int(d_o)
        di = canonical_ne(op_i, "i32") if d_i is None else int(d_i)
        out = np.empty(n, np.int32)
        _check(lib().oracle_segred2_i32(_ptr(x), _ptr(out), n, m, k, OPS[op_o], OPS[op_i], MAPS[f], _i32(do), _i32(di)))
        return out
    do = canonical_ne(op_o, "f32") if d_o is None else float(np.float32(d_o))
    di = canonical_ne(op_i, "f32") if d_i is None else float(np.float32(d_i))
    out = np.empty(n, np.float64)
    _check(lib().oracle_segred2_f32(_ptr(x), _ptr(out), n, m, k, OPS[op_o], OPS[op_i], MAPS[f], do, di))
    return out
