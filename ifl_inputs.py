"""Seeded synthetic input generators shared by the tests, the oracle legs and
bench.py.  This module holds none of the method's arithmetic -- only a
counter-based hash (splitmix64) and the value distributions of DESIGN.md's
input recipe, so the same element comes out on the CPU and on the GPU:

    h(seed, i) = splitmix64(i + (seed << 40)),   i = global flattened index

    I32_FULL    = (int32)(h >> 32)                 exercises wrap-around
    I32_SMALL   = ((h >> 11) % 2001) - 1000
    F32_UNIT    = (h >> 40) * 2^-24                in [0, 1), exact in f32
    F32_SIGNED  = 2 * F32_UNIT - 1                 in [-1, 1), never -0
    F32_EXACT   = ((h >> 11) % 3) - 1              {-1, 0, 1}: every partial
                                                   sum is an exact f32 integer
    BF16_SIGNED = ((h >> 56) - 128) / 128          exact in bf16

Everything is computed with torch int64 ops (two's-complement wrapping
multiply, logical shifts by masking), so it runs on CPU or CUDA tensors.
"""
from __future__ import annotations

import torch

_M64 = (1 << 64) - 1


def _s64(v: int) -> int:
    v &= _M64
    return v - (1 << 64) if v >= (1 << 63) else v


_GAMMA = _s64(0x9E3779B97F4A7C15)
_MUL1 = _s64(0xBF58476D1CE4E5B9)
_MUL2 = _s64(0x94D049BB133111EB)


def _lsr(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def splitmix64(idx: torch.Tensor) -> torch.Tensor:
    z = idx + _GAMMA
    z = (z ^ _lsr(z, 30)) * _MUL1
    z = (z ^ _lsr(z, 27)) * _MUL2
    return z ^ _lsr(z, 31)


def hash_range(seed: int, start: int, count: int, device="cpu") -> torch.Tensor:
    idx = torch.arange(start, start + count, dtype=torch.int64, device=device)
    return splitmix64(idx + (int(seed) << 40))


def _chunks(count: int, chunk: int = 1 << 24):
    s = 0
    while s < count:
        yield s, min(chunk, count - s)
        s += chunk


def generate(dist: str, seed: int, count: int, device="cpu", start: int = 0,
             out: torch.Tensor | None = None) -> torch.Tensor:
    """Return `count` elements of distribution `dist` for global indices
    [start, start+count).  Chunked so 2^30-element inputs fit in memory."""
    dt = {"I32_FULL": torch.int32, "I32_SMALL": torch.int32, "F32_UNIT": torch.float32,
          "F32_SIGNED": torch.float32, "F32_EXACT": torch.float32,
          "BF16_SIGNED": torch.bfloat16}[dist]
    if out is None:
        out = torch.empty(count, dtype=dt, device=device)
    for s, c in _chunks(count):
        h = hash_range(seed, start + s, c, device)
        if dist == "I32_FULL":
            v = _lsr(h, 32)
            v = torch.where(v >= (1 << 31), v - (1 << 32), v).to(torch.int32)
        elif dist == "I32_SMALL":
            v = (_lsr(h, 11) % 2001 - 1000).to(torch.int32)
        elif dist == "F32_UNIT":
            v = _lsr(h, 40).to(torch.float32) * (2.0 ** -24)
        elif dist == "F32_SIGNED":
            v = _lsr(h, 40).to(torch.float32) * (2.0 ** -23) - 1.0
        elif dist == "F32_EXACT":
            v = (_lsr(h, 11) % 3 - 1).to(torch.float32)
        else:  # BF16_SIGNED
            v = ((_lsr(h, 56) - 128).to(torch.float32) / 128.0).to(torch.bfloat16)
        out[s:s + c] = v
    return out


def matrix(dist: str, seed: int, n: int, m: int, device="cpu") -> torch.Tensor:
    return generate(dist, seed, n * m, device).view(n, m)


def tridag_system(seed: int, S: int, L: int, coef_rows: int, device="cpu"):
    """LocVolCalib-like diagonally dominant systems (DESIGN.md recipe):
    a, c ~ -U(0, 0.5); b = 1 + |a| + |c| + U(0, 1); y ~ U(-1, 1).
    Coefficients are [coef_rows][L], shared across the outer numS map."""
    u = lambda k, cnt: generate("F32_UNIT", seed * 16 + k, cnt, device)
    a = (-0.5 * u(0, coef_rows * L)).view(coef_rows, L)
    c = (-0.5 * u(1, coef_rows * L)).view(coef_rows, L)
    b = (1.0 + a.abs() + c.abs() + u(2, coef_rows * L).view(coef_rows, L))
    y = generate("F32_SIGNED", seed * 16 + 3, S * L, device).view(S, L)
    return a.contiguous(), b.contiguous(), c.contiguous(), y


LVC_DATASETS = {  # (numS, numT, numX, numY)
    "small": (16, 256, 32, 256),
    "medium": (128, 64, 256, 32),
    "large": (256, 64, 256, 256),
}


def lvc_problem(seed: int, numS: int, numX: int, numY: int, device="cpu"):
    """Inputs of the LocVolCalib loop (Fig 6a), DESIGN.md recipe:
    per site, coefficient rows a, c ~ -U(0, 0.5), b = 1 + |a| + |c| (the
    implicit diffusion step I - dt*D: interior rows sum to 1, so repeated
    solves neither blow up nor underflow over numT steps); x-site
    coefficients [numX][numY], y-site [numY][numX]; xsss [numS][numX][numY]
    and ysss [numS][numY][numX] ~ U(-1, 1)."""
    u = lambda k, cnt: generate("F32_UNIT", seed * 16 + k, cnt, device)

    def site(k0, R, L):
        a = (-0.5 * u(k0, R * L)).view(R, L)
        c = (-0.5 * u(k0 + 1, R * L)).view(R, L)
        b = 1.0 + a.abs() + c.abs()
        return a.contiguous(), b.contiguous(), c.contiguous()

    ax, bx, cx = site(0, numX, numY)
    ay, by, cy = site(2, numY, numX)
    xsss = generate("F32_SIGNED", seed * 16 + 4, numS * numX * numY, device).view(numS, numX, numY)
    ysss = generate("F32_SIGNED", seed * 16 + 5, numS * numY * numX, device).view(numS, numY, numX)
    return (ax, bx, cx), (ay, by, cy), xsss, ysss


def irregular_offsets(seed: int, n: int, mean: float, alpha: float = 1.5, max_len: int | None = None):
    """Segment descriptor for irregular nested parallelism (DESIGN.md
    recipe): n segment lengths from a Pareto-like heavy tail with the given
    mean (power-law degree distributions of sparse / graph workloads):
    len_i = floor(mean * (alpha - 1) / alpha * u_i^(-1/alpha)), u_i ~ U(0, 1],
    capped at max_len; about (1 - (alpha-1)/alpha * mean)-fraction of short
    and some empty segments at small means.  Returns int64 offsets [n + 1]."""
    import numpy as np
    u = 1.0 - generate("F32_UNIT", seed, n).double().numpy()  # (0, 1]
    lens = np.floor(mean * (alpha - 1) / alpha * u ** (-1.0 / alpha)).astype(np.int64)
    if max_len is not None:
        lens = np.minimum(lens, max_len)
    off = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    return off
