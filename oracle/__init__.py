"""oracle — ctypes front-end of the plain C CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this package.  The
product path (paper_conf_sc_nguyensckd10_b200) never imports it and shares
no code with it.  See oracle.c's header for what it computes and which
passage of /root/reference/PAPER.md each function follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, -O2 -ffp-contract=off, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        for sfx in ("f32", "f64"):
            fn = getattr(L, f"oracle_st7_{sfx}")
            fn.argtypes = [P, P, ctypes.c_long, ctypes.c_long, ctypes.c_long,
                           ctypes.c_double, ctypes.c_double, ctypes.c_int]
            fn.restype = ctypes.c_int
            fn = getattr(L, f"oracle_st27_{sfx}")
            fn.argtypes = [P, P, ctypes.c_long, ctypes.c_long, ctypes.c_long] + [ctypes.c_double] * 4 + \
                [ctypes.c_int]
            fn.restype = ctypes.c_int
            fn = getattr(L, f"oracle_st13_{sfx}")
            fn.argtypes = [P, P, ctypes.c_long, ctypes.c_long, ctypes.c_long] + [ctypes.c_double] * 3 + \
                [ctypes.c_int]
            fn.restype = ctypes.c_int
            fn = getattr(L, f"oracle_lbm_{sfx}")
            fn.argtypes = [P, P, P, ctypes.c_long, ctypes.c_long, ctypes.c_long,
                           ctypes.c_double, ctypes.c_int, ctypes.c_double, ctypes.c_double,
                           ctypes.c_double, ctypes.c_int]
            fn.restype = ctypes.c_int
            fn = getattr(L, f"oracle_feq_{sfx}")
            fn.argtypes = [ctypes.c_double] * 4 + [P]
            fn.restype = None
        L.oracle_d3q19_tables.argtypes = [P] * 5
        L.oracle_d3q19_tables.restype = None
        L.oracle_num_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _sfx(dtype) -> str:
    dt = np.dtype(dtype)
    if dt == np.float32:
        return "f32"
    if dt == np.float64:
        return "f64"
    raise ValueError(dt)


def st7(A0: np.ndarray, alpha: float, beta: float, T: int) -> np.ndarray:
    """T Jacobi sweeps of the 7-point stencil, Dirichlet shell."""
    A0 = np.ascontiguousarray(A0)
    nz, ny, nx = A0.shape
    out = np.empty_like(A0)
    rc = getattr(lib(), f"oracle_st7_{_sfx(A0.dtype)}")(
        A0.ctypes.data, out.ctypes.data, nx, ny, nz, alpha, beta, T)
    if rc != 0:
        raise RuntimeError(f"oracle_st7 rc={rc}")
    return out


def st27(A0: np.ndarray, alpha: float, beta: float, gamma: float, delta: float, T: int) -> np.ndarray:
    """T Jacobi sweeps of the 27-point stencil (weights centre/face/edge/corner), Dirichlet shell."""
    A0 = np.ascontiguousarray(A0)
    nz, ny, nx = A0.shape
    out = np.empty_like(A0)
    rc = getattr(lib(), f"oracle_st27_{_sfx(A0.dtype)}")(
        A0.ctypes.data, out.ctypes.data, nx, ny, nz, alpha, beta, gamma, delta, T)
    if rc != 0:
        raise RuntimeError(f"oracle_st27 rc={rc}")
    return out


def st13(A0: np.ndarray, alpha: float, beta: float, gamma: float, T: int) -> np.ndarray:
    """T Jacobi sweeps of the radius-2 13-point star (general R of §V; X25),
    Dirichlet shell 2 points thick (X26)."""
    A0 = np.ascontiguousarray(A0)
    nz, ny, nx = A0.shape
    out = np.empty_like(A0)
    rc = getattr(lib(), f"oracle_st13_{_sfx(A0.dtype)}")(
        A0.ctypes.data, out.ctypes.data, nx, ny, nz, alpha, beta, gamma, T)
    if rc != 0:
        raise RuntimeError(f"oracle_st13 rc={rc}")
    return out


def lbm(f0: np.ndarray, flags: np.ndarray, omega: float, T: int,
        u_lid=(0.05, 0.0, 0.0), periodic: bool = False) -> np.ndarray:
    """T D3Q19 push steps, BGK, bounce-back / moving lid."""
    f0 = np.ascontiguousarray(f0)
    flags = np.ascontiguousarray(flags, dtype=np.uint8)
    _, nz, ny, nx = f0.shape
    assert f0.shape[0] == 19 and flags.shape == (nz, ny, nx)
    out = np.empty_like(f0)
    rc = getattr(lib(), f"oracle_lbm_{_sfx(f0.dtype)}")(
        f0.ctypes.data, out.ctypes.data, flags.ctypes.data, nx, ny, nz, omega, T,
        u_lid[0], u_lid[1], u_lid[2], 1 if periodic else 0)
    if rc != 0:
        raise RuntimeError(f"oracle_lbm rc={rc}")
    return out


def feq(rho: float, ux: float, uy: float, uz: float, dtype=np.float64) -> np.ndarray:
    out = np.empty(19, dtype=dtype)
    getattr(lib(), f"oracle_feq_{_sfx(dtype)}")(rho, ux, uy, uz, out.ctypes.data)
    return out


def d3q19_tables():
    arrs = [np.zeros(19, dtype=np.int32) for _ in range(5)]
    lib().oracle_d3q19_tables(*[a.ctypes.data for a in arrs])
    ex, ey, ez, wden, opp = arrs
    return np.stack([ex, ey, ez], axis=1), wden, opp


def num_threads() -> int:
    return int(lib().oracle_num_threads())
