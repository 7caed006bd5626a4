"""stgen — seeded, counter-based synthetic inputs shared by the oracle tests,
the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no stencil, no collision,
no streaming).  It only turns (seed, global linear index) into numbers, plus
the geometry/initial-condition recipes DESIGN.md §"Input recipe" states:

* value(i) = splitmix64(seed XOR (i * 0x9E3779B97F4A7C15))
  where i is the GLOBAL linear index ``(z*ny + y)*nx + x`` (and, for LBM,
  ``pop*(nx*ny*nz) + cell``), so a Z-slab on rank r is generated
  independently and bit-identically to the same planes of the full grid.
* FP32 = (r >> 40) * 2^-24  (top 24 bits), FP64 = (r >> 11) * 2^-53 — exact
  conversions, so the same u64 stream gives the same value on every host.

Geometry recipe for the lid-driven cavity (BASELINE.json configs[2]/[4]):
flags[z][y][x] = 0 FLUID, 1 WALL (half-way bounce-back), 2 LID (moving wall);
the plane y = ny-1 is LID (all x, z — edges included), every other shell cell
is WALL (reading X14).

The D3Q19 weights appear here ONLY as the initial condition "fluid at rest,
rho = 1" (f_i = w_i) and as the centre of the random-pop recipe; they are the
textbook values 1/3, 1/18, 1/36 (reading X10) in the order of the
velocity table of DESIGN.md.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

FLUID, WALL, LID = 0, 1, 2

# textbook D3Q19 weights, velocity order 0; ±x,±y,±z; 7..18 (X10)
D3Q19_W = (1.0 / 3.0,) + (1.0 / 18.0,) * 6 + (1.0 / 36.0,) * 12

_CHUNK = 1 << 24


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (all arithmetic mod 2^64)."""
    with np.errstate(over="ignore"):
        z = x + GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def u64_at(seed: int, idx: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        return splitmix64(np.uint64(seed) ^ (idx.astype(np.uint64) * GOLDEN))


def uniform01(seed: int, start: int, count: int, dtype) -> np.ndarray:
    """U[0,1) for global indices start .. start+count-1, exact conversion."""
    dtype = np.dtype(dtype)
    out = np.empty(count, dtype=dtype)
    for off in range(0, count, _CHUNK):
        n = min(_CHUNK, count - off)
        idx = np.arange(start + off, start + off + n, dtype=np.uint64)
        r = u64_at(seed, idx)
        if dtype == np.float32:
            out[off:off + n] = (r >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)
        elif dtype == np.float64:
            out[off:off + n] = (r >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
        else:
            raise ValueError(f"unsupported dtype {dtype}")
    return out


def grid7(nx: int, ny: int, nz: int, seed: int, dtype, z0: int = 0, nzl: int | None = None) -> np.ndarray:
    """7-point input grid A0[z][y][x] ~ U[0,1) including the Dirichlet shell.

    ``z0``/``nzl`` select planes z0 .. z0+nzl-1 of the global grid (Z-slab)."""
    nzl = nz - z0 if nzl is None else nzl
    plane = nx * ny
    return uniform01(seed, z0 * plane, nzl * plane, dtype).reshape(nzl, ny, nx)


def cavity_flags(nx: int, ny: int, nz: int, z0: int = 0, nzl: int | None = None) -> np.ndarray:
    """Lid-driven cavity flags (uint8, [z][y][x]); lid = plane y = ny-1."""
    nzl = nz - z0 if nzl is None else nzl
    f = np.zeros((nzl, ny, nx), dtype=np.uint8)
    f[:, 0, :] = WALL
    f[:, :, 0] = WALL
    f[:, :, nx - 1] = WALL
    zs = np.arange(z0, z0 + nzl)
    f[zs == 0] = WALL
    f[zs == nz - 1] = WALL
    f[:, ny - 1, :] = LID
    return f


def periodic_fluid_flags(nx: int, ny: int, nz: int) -> np.ndarray:
    return np.zeros((nz, ny, nx), dtype=np.uint8)


def lbm_rest(nx: int, ny: int, nz: int, dtype, nzl: int | None = None) -> np.ndarray:
    """f_i = w_i everywhere (rho = 1, u = 0), SoA [19][z][y][x]."""
    nzl = nz if nzl is None else nzl
    f = np.empty((19, nzl, ny, nx), dtype=dtype)
    for i in range(19):
        f[i] = np.asarray(D3Q19_W[i], dtype=dtype)
    return f


def lbm_random(nx: int, ny: int, nz: int, seed: int, dtype, amp: float = 0.1,
               z0: int = 0, nzl: int | None = None) -> np.ndarray:
    """f_i = w_i * (1 + amp*(2U-1)), U keyed by the global (pop, cell) index."""
    dtype = np.dtype(dtype)
    nzl = nz - z0 if nzl is None else nzl
    ncell = nx * ny * nz
    plane = nx * ny
    f = np.empty((19, nzl, ny, nx), dtype=dtype)
    for i in range(19):
        u = uniform01(seed, i * ncell + z0 * plane, nzl * plane, dtype).reshape(nzl, ny, nx)
        w = dtype.type(D3Q19_W[i])
        f[i] = w * (dtype.type(1) + dtype.type(amp) * (dtype.type(2) * u - dtype.type(1)))
    return f
