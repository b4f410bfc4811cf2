"""B200-native incremental-flattening hot path (Henriksen et al., PPoPP'19).

Thin Python binding over the C ABI of ``include/ifl.h`` (``libifl.so``, built
in-tree for sm_100a by ``build.py``).  The binding only marshals arguments:
torch supplies device memory and the current CUDA stream; every step of the
path runs in the library's CUDA kernels.  There is no CPU fallback: if
``libifl.so`` is missing or no CUDA device is present the calls raise.

Functions keep the C names:
    ifl_segred, ifl_segscan, ifl_redomap2, ifl_tridag, ifl_select,
    ifl_set_thresholds, ifl_get_thresholds, ifl_tune, ...
``segred`` / ``segscan`` / ``redomap2`` / ``tridag`` are the tensor-level
conveniences (they also accept pinned host tensors: copy in, compute, copy
out -- the end-to-end path bench.py times).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("IFL_LIB_PATH") or os.path.join(_PKG, "libifl.so")  # override: experiment builds

IFL_OK, IFL_EINVAL, IFL_EUNSUPPORTED, IFL_EWORKSPACE, IFL_ENOTFIT, IFL_ECUDA = 0, -1, -2, -3, -4, -5
DTYPES = {"i32": 0, "f32": 1, "bf16": 2}
OPS = {"sum": 0, "prod": 1, "min": 2, "max": 3, "and": 4, "or": 5, "xor": 6}
MAPS = {"id": 0, "sq": 1, "abs": 2}
VERSIONS = {"auto": -1, "top": 0, "middle": 1, "flat": 2, "outer": 3, "row_top": 4, "row_middle": 5, "cluster": 6}
VERSION_NAMES = {v: k for k, v in VERSIONS.items()}
SITES = ("segred.b4", "segscan.b4", "redomap2.f32", "redomap2.bf16", "tridag", "lvc", "colred.b4", "colscan.b4",
         "segred.irr", "segscan.irr", "segarg.b4", "redomap2.f32.row", "redomap2.bf16.row",
         "segred2.b4", "segred.b4.cl", "segscan.b4.cl", "segred.b4.midg", "segscan.b4.midg")

_TORCH_DT = {torch.int32: "i32", torch.float32: "f32", torch.bfloat16: "bf16"}


class IflError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"ifl error {code}: {msg}")
        self.code = code


class ifl_choice(ctypes.Structure):
    _fields_ = [("version", ctypes.c_int), ("par_top", ctypes.c_int64), ("par_mid", ctypes.c_int64),
                ("t_top", ctypes.c_int64), ("t_intra", ctypes.c_int64)]


@dataclass
class Choice:
    version: str
    par_top: int
    par_mid: int
    t_top: int
    t_intra: int


_lib = None
_i64, _int, _vp, _sz = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
_SIGS = {
    "ifl_segred": ([_vp, _vp, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segscan": ([_vp, _vp, _i64, _i64, _int, _int, _int, _vp, _int, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segscan_seeded": ([_vp, _vp, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_colred": ([_vp, _vp, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_colscan": ([_vp, _vp, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segred2": ([_vp, _vp, _i64, _i64, _i64, _int, _int, _int, _int, _vp, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segarg": ([_vp, _vp, _vp, _i64, _i64, _int, _int, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segred_irr": ([_vp, _vp, _vp, _i64, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_segscan_irr": ([_vp, _vp, _vp, _i64, _i64, _i64, _int, _int, _int, _vp, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_irr_inspect": ([_vp, _i64, _i64, _vp, _vp, _vp], _int),
    "ifl_redomap2": ([_vp, _vp, _vp, _i64, _i64, _i64, _int, _int, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_tridag": ([_vp, _vp, _vp, _vp, _vp, _i64, _i64, _i64, _int, _vp, _sz, _vp, _vp], _int),
    "ifl_lvc": ([_vp] * 8 + [_i64] * 4 + [_int, _vp, _sz, _vp, _vp], _int),
    "ifl_workspace_bytes": ([ctypes.c_char_p, _i64, _i64, _i64, _int, _int], _sz),
    "ifl_workspace_init": ([_vp, _sz, _vp], _int),
    "ifl_select": ([ctypes.c_char_p, _i64, _i64, _i64, _vp], _int),
    "ifl_set_thresholds": ([ctypes.c_char_p, _i64, _i64], _int),
    "ifl_get_thresholds": ([ctypes.c_char_p, _vp, _vp], _int),
    "ifl_reset_thresholds": ([], _int),
    "ifl_set_par_mode": ([_int], _int),
    "ifl_get_par_mode": ([], _int),
    "ifl_save_thresholds": ([ctypes.c_char_p], _int),
    "ifl_load_thresholds": ([ctypes.c_char_p], _int),
    "ifl_tune": ([ctypes.c_char_p, _vp, _int, _int, _int, _vp, _sz, _vp, _vp, _vp, _vp], _int),
    "ifl_tune_scratch_bytes": ([ctypes.c_char_p, _vp, _int], _sz),
    "ifl_tune_search": ([_vp, _vp, _vp, _int, _int, _vp, _vp, _vp], _int),
    "ifl_tune_search_chain": ([_vp, _vp, _int, _int, _int, _vp, _vp], _int),
    "ifl_last_error": ([], ctypes.c_char_p),
    "ifl_build_info": ([], ctypes.c_char_p),
}
EXPORTED = tuple(_SIGS)


def lib() -> ctypes.CDLL:
    """Load libifl.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_ppopp_henriksenteo19_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        for name, (argt, rest) in _SIGS.items():
            fn = getattr(L, name)
            fn.argtypes = argt
            fn.restype = rest
        _lib = L
    return _lib


def _check(rc: int, what: str):
    if rc != IFL_OK:
        raise IflError(rc, f"{what}: {lib().ifl_last_error().decode()}")


def _stream(s=None) -> int:
    if s is None:
        s = torch.cuda.current_stream()
    return s.cuda_stream


def _b(s: str) -> bytes:
    return s.encode()


# ------------------------------------------------------------------ selector


def select(site: str, n: int, m: int, p: int = 0) -> Choice:
    c = ifl_choice()
    _check(lib().ifl_select(_b(site), n, m, p, ctypes.byref(c)), "ifl_select")
    return Choice(VERSION_NAMES[c.version], c.par_top, c.par_mid, c.t_top, c.t_intra)


def set_thresholds(site: str, t_top: int, t_intra: int):
    _check(lib().ifl_set_thresholds(_b(site), int(t_top), int(t_intra)), "ifl_set_thresholds")


def get_thresholds(site: str):
    a, b = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().ifl_get_thresholds(_b(site), ctypes.byref(a), ctypes.byref(b)), "ifl_get_thresholds")
    return a.value, b.value


def reset_thresholds():
    _check(lib().ifl_reset_thresholds(), "ifl_reset_thresholds")


def set_par_mode(mode: int):
    _check(lib().ifl_set_par_mode(int(mode)), "ifl_set_par_mode")


def get_par_mode() -> int:
    return lib().ifl_get_par_mode()


def save_thresholds(path: str):
    _check(lib().ifl_save_thresholds(_b(path)), "ifl_save_thresholds")


def load_thresholds(path: str):
    _check(lib().ifl_load_thresholds(_b(path)), "ifl_load_thresholds")


def workspace_bytes(entry: str, n: int, m: int, p: int = 0, dt: str = "f32", version: str = "auto") -> int:
    return lib().ifl_workspace_bytes(_b(entry), n, m, p, DTYPES[dt], VERSIONS[version])


def tune_search(par_top, par_mid, cost_table, cost: int = 0):
    """Pure host threshold search over a cost table [[t_top, t_mid, t_flat], ...]."""
    import numpy as np
    pt = np.ascontiguousarray(par_top, dtype=np.int64)
    pm = np.ascontiguousarray(par_mid, dtype=np.int64)
    ct = np.ascontiguousarray(cost_table, dtype=np.float64).reshape(-1)
    a, b, npaths = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int()
    _check(lib().ifl_tune_search(pt.ctypes.data, pm.ctypes.data, ct.ctypes.data, len(pt), cost,
                                 ctypes.byref(a), ctypes.byref(b), ctypes.byref(npaths)), "ifl_tune_search")
    return a.value, b.value, npaths.value


def tune_search_chain(par, cost_table, cost: int = 0):
    """Chain (Fig 5) search: par [nshapes][G], cost_table [nshapes][G+1] ->
    (thresholds [G], distinct paths evaluated)."""
    import numpy as np
    pa = np.ascontiguousarray(par, dtype=np.int64)
    ct = np.ascontiguousarray(cost_table, dtype=np.float64)
    ns, G = pa.shape
    th = np.zeros(G, np.int64)
    npaths = ctypes.c_int()
    _check(lib().ifl_tune_search_chain(pa.ctypes.data, ct.ctypes.data, ns, G, cost, th.ctypes.data,
                                       ctypes.byref(npaths)), "ifl_tune_search_chain")
    return [int(t) for t in th], npaths.value


# ------------------------------------------------------------- workspaces

_WS: dict = {}


def workspace(nbytes: int, device=None, key: str = "default", stream=None) -> torch.Tensor:
    """A zero-initialised, reusable device workspace (the flat kernels leave it
    re-armed for the next call, so it is zeroed only when first allocated).
    One cache per (device, key, stream): the conveniences below key it by entry
    point, so segred partials never land in a segscan status region, and two
    streams never share one workspace (ifl.h forbids concurrent use)."""
    if nbytes == 0:
        return None
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    k = (dev, key, 0 if stream is None else int(stream))
    w = _WS.get(k)
    if w is None or w.numel() < nbytes:
        w = torch.zeros(max(nbytes, 1 << 20), dtype=torch.uint8, device=dev)
        _WS[k] = w
    return w


def _ptr(t):
    return 0 if t is None else t.data_ptr()


def _ne_buf(ne, dt: str):
    if ne is None:
        return None
    if dt == "i32":
        return ctypes.byref(ctypes.c_int32(int(ne)))
    return ctypes.byref(ctypes.c_float(float(ne)))


def _choice_out(c: ifl_choice) -> Choice:
    return Choice(VERSION_NAMES.get(c.version, str(c.version)), c.par_top, c.par_mid, c.t_top, c.t_intra)


# ---------------------------------------------------------- segred / segscan


def _seg(scan: bool, x: torch.Tensor, op: str, f: str, ne, version: str, out, ws, stream, return_choice,
         seed=None, reverse=False):
    host = not x.is_cuda
    if host:  # end-to-end path: pinned host -> device -> host
        xd = x.to("cuda", non_blocking=True)
        sd = None if seed is None else seed.to("cuda", non_blocking=True)
        r = _seg(scan, xd, op, f, ne, version, None, ws, stream, return_choice, sd, reverse)
        if return_choice:
            r, c = r
        o = torch.empty(r.shape, dtype=r.dtype, pin_memory=True) if out is None else out
        o.copy_(r, non_blocking=True)
        torch.cuda.current_stream().synchronize()
        return (o, c) if return_choice else o
    if x.dim() != 2:
        raise ValueError("expected an [n][m] tensor")
    if not x.is_contiguous():
        raise ValueError("input must be contiguous row-major")
    dt = _TORCH_DT.get(x.dtype)
    if dt not in ("i32", "f32"):
        raise TypeError(f"unsupported dtype {x.dtype}")
    n, m = x.shape
    if out is None:
        out = torch.empty((n, m) if scan else (n,), dtype=x.dtype, device=x.device)
    entry = "segscan" if scan else "segred"
    wb = lib().ifl_workspace_bytes(_b(entry), n, m, 0, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, x.device, entry, _stream(stream))
    c = ifl_choice()
    args = (x.data_ptr(), out.data_ptr(), n, m, DTYPES[dt], OPS[op], MAPS[f], _ne_buf(ne, dt))
    tail = (VERSIONS[version], _ptr(ws), 0 if ws is None else ws.numel() * ws.element_size(),
            _stream(stream), ctypes.byref(c))
    if seed is not None:
        if seed.dtype != x.dtype or seed.numel() != n or not seed.is_contiguous() or seed.device != x.device:
            raise ValueError("seed must be a contiguous [n] tensor of x's dtype on x's device")
        rc = lib().ifl_segscan_seeded(*args[:7], seed.data_ptr(), *tail)
        entry = "segscan_seeded"
    elif scan:
        rc = lib().ifl_segscan(*args, 1 if reverse else 0, *tail)
    else:
        rc = lib().ifl_segred(*args, *tail)
    _check(rc, "ifl_" + entry)
    return (out, _choice_out(c)) if return_choice else out


def segred(x, op="sum", f="id", ne=None, version="auto", out=None, ws=None, stream=None, return_choice=False):
    """out[i] = ne (+) f(x[i,0]) (+) ... (+) f(x[i,m-1])."""
    return _seg(False, x, op, f, ne, version, out, ws, stream, return_choice)


def segscan(x, op="sum", f="id", ne=None, version="auto", out=None, ws=None, stream=None, return_choice=False,
            seed=None, reverse=False):
    """Inclusive per-row scanomap (example P:116).  ``seed``
    (an [n] tensor) replaces ne row by row: out[i,j] = seed[i] (+) f(x[i,0])
    (+) ... (+) f(x[i,j]) -- the carry-in of a column block (ifl_segscan_seeded).
    ``reverse``: out[i,j] = ne (+) f(x[i,m-1]) (+) ... (+) f(x[i,j])."""
    if seed is not None and ne is not None:
        raise ValueError("pass either ne or seed")
    if seed is not None and reverse:
        raise ValueError("seeded scans run forward only")
    return _seg(True, x, op, f, ne, version, out, ws, stream, return_choice, seed, reverse)


# ----------------------------------------------------------- colred / colscan


def _col(scan: bool, x: torch.Tensor, op: str, f: str, ne, version: str, out, ws, stream, return_choice):
    if x.dim() != 2 or not x.is_contiguous() or not x.is_cuda:
        raise ValueError("expected a contiguous [n][m] CUDA tensor")
    dt = _TORCH_DT.get(x.dtype)
    if dt not in ("i32", "f32"):
        raise TypeError(f"unsupported dtype {x.dtype}")
    n, m = x.shape
    if out is None:
        out = torch.empty((n, m) if scan else (m,), dtype=x.dtype, device=x.device)
    entry = "colscan" if scan else "colred"
    wb = lib().ifl_workspace_bytes(_b(entry), n, m, 0, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, x.device, entry, _stream(stream))
    c = ifl_choice()
    fn = lib().ifl_colscan if scan else lib().ifl_colred
    rc = fn(x.data_ptr(), out.data_ptr(), n, m, DTYPES[dt], OPS[op], MAPS[f], _ne_buf(ne, dt), VERSIONS[version],
            _ptr(ws), 0 if ws is None else ws.numel() * ws.element_size(), _stream(stream), ctypes.byref(c))
    _check(rc, "ifl_" + entry)
    return (out, _choice_out(c)) if return_choice else out


def colred(x, op="sum", f="id", ne=None, version="auto", out=None, ws=None, stream=None, return_choice=False):
    """out[j] = ne (+) f(x[0,j]) (+) ... (+) f(x[n-1,j]) -- G4's column reduction."""
    return _col(False, x, op, f, ne, version, out, ws, stream, return_choice)


def colscan(x, op="sum", f="id", ne=None, version="auto", out=None, ws=None, stream=None, return_choice=False):
    """out[i,j] = ne (+) f(x[0,j]) (+) ... (+) f(x[i,j]) -- column-wise inclusive scan (G4 with scan)."""
    return _col(True, x, op, f, ne, version, out, ws, stream, return_choice)


# ------------------------------------------------------------- segred2


def segred2(x, op_o="sum", op_i="max", f="id", ne_o=None, ne_i=None, version="auto", out=None, ws=None,
            stream=None, return_choice=False):
    """Nested reduce over an [n][m][k] tensor (G9's e_rec):
    out[i] = ne_o (+)_j (ne_i (x)_q f(x[i,j,q])), (+) = op_o, (x) = op_i."""
    if x.dim() != 3 or not x.is_contiguous() or not x.is_cuda:
        raise ValueError("expected a contiguous [n][m][k] CUDA tensor")
    dt = _TORCH_DT.get(x.dtype)
    if dt not in ("i32", "f32"):
        raise TypeError(f"unsupported dtype {x.dtype}")
    n, m, k = x.shape
    if out is None:
        out = torch.empty(n, dtype=x.dtype, device=x.device)
    wb = lib().ifl_workspace_bytes(b"segred2", n, m, k, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, x.device, "segred2", _stream(stream))
    c = ifl_choice()
    rc = lib().ifl_segred2(x.data_ptr(), out.data_ptr(), n, m, k, DTYPES[dt], OPS[op_o], OPS[op_i], MAPS[f],
                           _ne_buf(ne_o, dt), _ne_buf(ne_i, dt), VERSIONS[version], _ptr(ws),
                           0 if ws is None else ws.numel() * ws.element_size(), _stream(stream), ctypes.byref(c))
    _check(rc, "ifl_segred2")
    return (out, _choice_out(c)) if return_choice else out


# -------------------------------------------------------------- segarg


def segarg(x, which="min", version="auto", out=None, ws=None, stream=None, return_choice=False):
    """Per-row (value, index) of the first minimum / maximum -- the
    tuple-valued reduction (argmin of NN).  Returns (val, idx)."""
    if x.dim() != 2 or not x.is_contiguous() or not x.is_cuda:
        raise ValueError("expected a contiguous [n][m] CUDA tensor")
    dt = _TORCH_DT.get(x.dtype)
    if dt not in ("i32", "f32"):
        raise TypeError(f"unsupported dtype {x.dtype}")
    n, m = x.shape
    val, idx = out if out is not None else (torch.empty(n, dtype=x.dtype, device=x.device),
                                            torch.empty(n, dtype=torch.int32, device=x.device))
    wb = lib().ifl_workspace_bytes(b"segarg", n, m, 0, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, x.device, "segarg", _stream(stream))
    c = ifl_choice()
    rc = lib().ifl_segarg(x.data_ptr(), val.data_ptr(), idx.data_ptr(), n, m, DTYPES[dt], 1 if which == "max" else 0,
                          VERSIONS[version], _ptr(ws), 0 if ws is None else ws.numel() * ws.element_size(),
                          _stream(stream), ctypes.byref(c))
    _check(rc, "ifl_segarg")
    return ((val, idx), _choice_out(c)) if return_choice else (val, idx)


# -------------------------------------------------------- irregular segments


def irr_inspect(offsets: torch.Tensor, total: int, stream=None) -> int:
    """Inspector: validate the descriptor and return the longest
    segment (synchronises the stream)."""
    ws = workspace(16, offsets.device, "irr_inspect")
    mx = ctypes.c_int64()
    _check(lib().ifl_irr_inspect(offsets.data_ptr(), offsets.numel() - 1, int(total), ws.data_ptr(), _stream(stream),
                                 ctypes.byref(mx)), "ifl_irr_inspect")
    return mx.value


def _irr(scan, x, offsets, op, f, ne, version, max_len, out, ws, stream, return_choice):
    if x.dim() != 1 or not x.is_contiguous() or not x.is_cuda:
        raise ValueError("expected a contiguous 1-D CUDA tensor of segment data")
    if offsets.dtype != torch.int64 or not offsets.is_contiguous() or offsets.device != x.device:
        raise ValueError("offsets must be a contiguous int64 tensor on x's device")
    dt = _TORCH_DT.get(x.dtype)
    if dt not in ("i32", "f32"):
        raise TypeError(f"unsupported dtype {x.dtype}")
    n, total = offsets.numel() - 1, x.numel()
    if out is None:
        out = torch.empty(total if scan else n, dtype=x.dtype, device=x.device)
    entry = "segscan_irr" if scan else "segred_irr"
    wb = lib().ifl_workspace_bytes(_b(entry), n, total, 0, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, x.device, entry, _stream(stream))
    c = ifl_choice()
    fn = lib().ifl_segscan_irr if scan else lib().ifl_segred_irr
    rc = fn(x.data_ptr(), out.data_ptr(), offsets.data_ptr(), n, total, int(max_len), DTYPES[dt], OPS[op], MAPS[f],
            _ne_buf(ne, dt), VERSIONS[version], _ptr(ws), 0 if ws is None else ws.numel() * ws.element_size(),
            _stream(stream), ctypes.byref(c))
    _check(rc, "ifl_" + entry)
    return (out, _choice_out(c)) if return_choice else out


def segred_irr(x, offsets, op="sum", f="id", ne=None, version="auto", max_len=0, out=None, ws=None, stream=None,
               return_choice=False):
    """out[i] = ne (+) f(x[offsets[i]]) (+) ... (+) f(x[offsets[i+1]-1]) (irregular segments)."""
    return _irr(False, x, offsets, op, f, ne, version, max_len, out, ws, stream, return_choice)


def segscan_irr(x, offsets, op="sum", f="id", ne=None, version="auto", max_len=0, out=None, ws=None, stream=None,
                return_choice=False):
    """Inclusive scan of every irregular segment."""
    return _irr(True, x, offsets, op, f, ne, version, max_len, out, ws, stream, return_choice)


# ------------------------------------------------------------------ redomap2


def redomap2(A, B, b_kmajor=True, version="auto", out=None, ws=None, stream=None, return_choice=False):
    """C = xss x yss as map-map-redomap.  B is transpose yss ([p][m])
    when b_kmajor, else yss ([m][p]).  A/B float32 or bfloat16; C float32."""
    if A.dtype != B.dtype or A.dtype not in (torch.float32, torch.bfloat16):
        raise TypeError("A and B must both be float32 or both bfloat16")
    if not (A.is_contiguous() and B.is_contiguous()):
        raise ValueError("A and B must be contiguous")
    n, m = A.shape
    p = B.shape[0] if b_kmajor else B.shape[1]
    dt = _TORCH_DT[A.dtype]
    if out is None:
        out = torch.empty((n, p), dtype=torch.float32, device=A.device)
    wb = lib().ifl_workspace_bytes(b"redomap2", n, m, p, DTYPES[dt], VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, A.device, "redomap2", _stream(stream))
    c = ifl_choice()
    rc = lib().ifl_redomap2(A.data_ptr(), B.data_ptr(), out.data_ptr(), n, m, p, DTYPES[dt], int(b_kmajor),
                            VERSIONS[version], _ptr(ws), 0 if ws is None else ws.numel(), _stream(stream),
                            ctypes.byref(c))
    _check(rc, "ifl_redomap2")
    return (out, _choice_out(c)) if return_choice else out


# -------------------------------------------------------------------- tridag


def tridag(a, b, c, y, version="auto", out=None, ws=None, stream=None, return_choice=False):
    """Batched tridiagonal solves; coefficients [R][L] shared by
    systems s with s % R == r."""
    S, L = y.shape
    R = a.shape[0]
    for t in (a, b, c, y):
        if t.dtype != torch.float32 or not t.is_contiguous():
            raise TypeError("tridag takes contiguous float32 tensors")
    if out is None:
        out = torch.empty_like(y)
    wb = lib().ifl_workspace_bytes(b"tridag", S, L, R, 1, VERSIONS[version])
    if ws is None and wb:
        ws = workspace(wb, y.device, "tridag", _stream(stream))
    ch = ifl_choice()
    rc = lib().ifl_tridag(a.data_ptr(), b.data_ptr(), c.data_ptr(), y.data_ptr(), out.data_ptr(), S, L, R,
                          VERSIONS[version], _ptr(ws), 0 if ws is None else ws.numel(), _stream(stream),
                          ctypes.byref(ch))
    _check(rc, "ifl_tridag")
    return (out, _choice_out(ch)) if return_choice else out


# ----------------------------------------------------------------------- lvc


def lvc(xsss, ysss, xcoef, ycoef, numT: int, version="auto", ws=None, stream=None, return_choice=False):
    """The LocVolCalib loop of Fig 6a, in place on xsss
    [numS][numX][numY] and ysss [numS][numY][numX]; xcoef = (a, b, c) each
    [numX][numY], ycoef = (a, b, c) each [numY][numX]."""
    numS, numX, numY = xsss.shape
    ts = (xsss, ysss) + tuple(xcoef) + tuple(ycoef)
    for t in ts:
        if t.dtype != torch.float32 or not t.is_contiguous() or not t.is_cuda:
            raise TypeError("lvc takes contiguous float32 CUDA tensors")
    if tuple(ysss.shape) != (numS, numY, numX):
        raise ValueError("ysss must be [numS][numY][numX]")
    wb = lib().ifl_workspace_bytes(b"lvc", numX, numY, 0, 1, -1)
    if ws is None and wb:
        ws = workspace(wb, xsss.device, "lvc", _stream(stream))
    ch = ifl_choice()
    rc = lib().ifl_lvc(*(t.data_ptr() for t in ts), numS, int(numT), numX, numY, VERSIONS[version], _ptr(ws),
                       0 if ws is None else ws.numel(), _stream(stream), ctypes.byref(ch))
    _check(rc, "ifl_lvc")
    return _choice_out(ch) if return_choice else None


# ---------------------------------------------------------------------- tuner


def tune(site: str, shapes, reps: int = 5, cost: int = 0, scratch: torch.Tensor | None = None, stream=None):
    """Offline tuner: time every forced version on the training
    shapes, exact search over the branching-tree paths, install thresholds.
    Returns (t_top, t_intra, cost_table[nshapes][3] in ms)."""
    import numpy as np
    sh = np.ascontiguousarray(shapes, dtype=np.int64)
    ns = sh.shape[0]
    need = lib().ifl_tune_scratch_bytes(_b(site), sh.ctypes.data, ns)
    if scratch is None or scratch.numel() < need:
        scratch = torch.zeros(need, dtype=torch.uint8, device="cuda")
    if sh.ndim != 2 or sh.shape[1] != (2 if site.startswith(("seg", "col")) else 4 if site == "lvc" else 3):
        raise ValueError(f"{site}: shapes must be tuples of the site's arity")
    nv = (5 if site.startswith("redomap2") else 4) if site.endswith(".tree") else 5 if site.endswith(".midg") else 3
    tbl = np.zeros(ns * nv, np.float64)
    a, b = ctypes.c_int64(), ctypes.c_int64()
    _check(lib().ifl_tune(_b(site), sh.ctypes.data, ns, reps, cost, scratch.data_ptr(), scratch.numel(),
                          _stream(stream), ctypes.byref(a), ctypes.byref(b), tbl.ctypes.data), "ifl_tune")
    return a.value, b.value, tbl.reshape(ns, nv)


def build_info() -> str:
    return lib().ifl_build_info().decode()
