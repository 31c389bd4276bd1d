"""Seeded synthetic field generator shared by the oracle harness and the CUDA path.

This module holds NO stencil arithmetic: it only turns (seed, array id, global
grid coordinate) into a pseudo-random number (SURVEY.md §8(d) "Synthetic
inputs", reading R19 in DESIGN.md).  Both sides of every parity test call it, so
the inputs are identical by construction; neither side's arithmetic lives here.

Generator (counter based, layout independent):

    key  = seed_mix(seed, array_id) ^ pack(i, j, k)
    bits = splitmix64(key)
    f64  = (bits >> 11) * 2**-53 * 2 - 1      exact in binary64, uniform [-1, 1)
    f32  = (bits >> 40) * 2**-24 * 2 - 1      exact in binary32, uniform [-1, 1)

(i, j, k) are GLOBAL interior coordinates (ghosts are negative or >= n), so a
z-slab of a decomposed grid receives exactly the values the undecomposed grid
holds there (pin P9 in SURVEY.md §8(c)).
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_BIAS = 1 << 20  # coordinates packed in 21-bit fields after biasing


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vigna's splitmix64 finaliser on a uint64 numpy array (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def seed_mix(seed: int, array_id: int) -> np.uint64:
    with np.errstate(over="ignore"):
        s = splitmix64(np.array([seed], dtype=np.uint64))[0]
        return np.uint64(s ^ (np.uint64(array_id + 1) * _GOLDEN))


def pack(i, j, k):
    i = np.asarray(i, dtype=np.int64) + _BIAS
    j = np.asarray(j, dtype=np.int64) + _BIAS
    k = np.asarray(k, dtype=np.int64) + _BIAS
    return ((k.astype(np.uint64) << np.uint64(42)) | (j.astype(np.uint64) << np.uint64(21))
            | i.astype(np.uint64))


def bits_to_unit(bits: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "f64":
        return (bits >> np.uint64(11)).astype(np.float64) * (2.0 ** -52) - 1.0
    if dtype == "f32":
        return ((bits >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -23)
                - np.float32(1.0)).astype(np.float32)
    raise ValueError(dtype)


def np_dtype(dtype: str):
    return {"f64": np.float64, "f32": np.float32}[dtype]


def field(seed: int, array_id: int, n: tuple, ghost: tuple, dtype: str,
          z_offset: int = 0, nz_alloc_extra: tuple = (0, 0)) -> np.ndarray:
    """Dense padded array [nz+2hz][ny+2hy][nx+2hx] (x fastest) of uniform [-1,1).

    n = (nx, ny, nz) interior size of THIS slab, ghost = (hx, hy, hz).
    z_offset = global z of local plane 0 (multi-rank slabs).
    nz_alloc_extra = extra ghost planes (below, above) beyond hz (deep halos).
    Element [k][j][i] holds the value at global (i - hx, j - hy, k - hz_lo + z_offset).
    """
    nx, ny, nz = n
    hx, hy, hz = ghost
    lo = hz + nz_alloc_extra[0]
    hi = hz + nz_alloc_extra[1]
    i = np.arange(-hx, nx + hx, dtype=np.int64)
    j = np.arange(-hy, ny + hy, dtype=np.int64)
    k = np.arange(-lo, nz + hi, dtype=np.int64) + z_offset
    key = pack(i[None, None, :], j[None, :, None], k[:, None, None])
    bits = splitmix64(key ^ seed_mix(seed, array_id))
    return bits_to_unit(bits, dtype)


def field_torch(seed: int, array_id: int, n: tuple, ghost: tuple, dtype: str,
                device, z_offset: int = 0, nz_alloc_extra: tuple = (0, 0)):
    """Same values as field(), generated with torch on `device` (for GPU-sized inputs).

    torch has no uint64 arithmetic on CUDA, so int64 is used with wrapping
    multiplication and logical right shifts emulated by masking.
    """
    import torch

    def u(v):  # python int -> int64 with the same bit pattern
        v &= (1 << 64) - 1
        return v - (1 << 64) if v >= (1 << 63) else v

    def lsr(x, s):
        return (x >> s) & ((1 << (64 - s)) - 1)

    def sm64(x):
        z = x + u(0x9E3779B97F4A7C15)
        z = (z ^ lsr(z, 30)) * u(0xBF58476D1CE4E5B9)
        z = (z ^ lsr(z, 27)) * u(0x94D049BB133111EB)
        return z ^ lsr(z, 31)

    nx, ny, nz = n
    hx, hy, hz = ghost
    lo = hz + nz_alloc_extra[0]
    hi = hz + nz_alloc_extra[1]
    mix = u(int(seed_mix(seed, array_id)))
    i = torch.arange(-hx, nx + hx, dtype=torch.int64, device=device) + _BIAS
    j = torch.arange(-hy, ny + hy, dtype=torch.int64, device=device) + _BIAS
    out_dtype = torch.float64 if dtype == "f64" else torch.float32
    out = torch.empty((nz + lo + hi, ny + 2 * hy, nx + 2 * hx), dtype=out_dtype, device=device)
    jk = (j << 21)[:, None] | i[None, :]
    for kk in range(nz + lo + hi):
        kg = kk - lo + z_offset + _BIAS
        key = (jk | (kg << 42)) ^ mix
        bits = sm64(key)
        if dtype == "f64":
            out[kk] = lsr(bits, 11).to(torch.float64) * (2.0 ** -52) - 1.0
        else:
            out[kk] = lsr(bits, 40).to(torch.float32) * (2.0 ** -23) - 1.0
    return out
