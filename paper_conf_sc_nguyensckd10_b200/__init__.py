"""paper_conf_sc_nguyensckd10_b200 — thin Python binding of libst35d.so.

Argument marshalling only: every step of the sweep runs in the library's
sm_100a kernels (include/st35d.h).  Names mirror the C ABI:
st_plan_create, st7_run, lbm_d3q19_run, st_destroy, ...

Buffers may be torch CUDA tensors (the fast path: the call enqueues kernels
on the plan stream and returns), or host numpy arrays / CPU tensors (the
library stages them through device memory and synchronises).  There is no
CPU fallback: without the built library or a CUDA device the calls raise.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("ST35D_LIB") or os.path.join(_HERE, "libst35d.so")   # override: A/B tuning builds

ST_F32, ST_F64 = 0, 1
ST_OK, ST_EINVAL, ST_ENOMEM, ST_ECUDA, ST_ENCCL, ST_EUNSUPPORTED = 0, -1, -2, -3, -4, -5
ST_FLUID, ST_WALL, ST_LID = 0, 1, 2
ST_MAX_DIM_T = 8
ST_OPT_LBM_BATCHED, ST_OPT_LBM_KERNEL, ST_OPT_OVERLAP, ST_OPT_PDL, ST_OPT_ST7_VARIANT, ST_OPT_ZCHUNK = 1, 2, 3, 4, 5, 6
ST_OPT_LBM_STAGES = 7
_ERRNAMES = {-1: "ST_EINVAL", -2: "ST_ENOMEM", -3: "ST_ECUDA", -4: "ST_ENCCL", -5: "ST_EUNSUPPORTED"}


class StError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{_ERRNAMES.get(code, code)}: {msg}")
        self.code = code


class st_plan_info(ctypes.Structure):
    _fields_ = [("tile_x", ctypes.c_int), ("tile_y", ctypes.c_int), ("out_x", ctypes.c_int),
                ("out_y", ctypes.c_int), ("tiles_x", ctypes.c_int), ("tiles_y", ctypes.c_int),
                ("ctas", ctypes.c_int), ("threads", ctypes.c_int), ("smem_bytes", ctypes.c_int),
                ("kappa", ctypes.c_double), ("kernel", ctypes.c_int), ("dim_t_sweep", ctypes.c_int),
                ("ring", ctypes.c_int)]


class st_autotune_report(ctypes.Structure):
    _fields_ = [("dim_T", ctypes.c_int), ("eta", ctypes.c_int), ("eta_nominal", ctypes.c_int),
                ("gamma", ctypes.c_double), ("Gamma_nominal", ctypes.c_double), ("Gamma_eff", ctypes.c_double),
                ("bw_dim1", ctypes.c_double), ("fp_deep", ctypes.c_double),
                ("tested", ctypes.c_int * ST_MAX_DIM_T), ("ms", ctypes.c_float * ST_MAX_DIM_T),
                ("capacity", ctypes.c_double * 3), ("tile_side", ctypes.c_int * 3), ("kappa", ctypes.c_double * 3)]


class st_slab_step(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int) for k in ("kind", "sweep", "depth", "src", "z_begin", "z_end", "async_", "grid_cap")]


ST_STEP_EXCHANGE, ST_STEP_SWEEP, ST_STEP_WAIT, ST_STEP_COPY = 0, 1, 2, 3


class st_blocking(ctypes.Structure):
    _fields_ = [("eta", ctypes.c_int), ("dim_bound", ctypes.c_double), ("dim", ctypes.c_int),
                ("kappa", ctypes.c_double)]


_lib = None

EXPORTS = ["st_plan_create", "st7_run", "st13_run", "st27_run", "lbm_d3q19_run", "st_destroy", "st_last_error", "st_last_status",
           "st_plan_set_stream", "st_plan_set_option", "st_plan_set_lbm_lid", "st_plan_set_bitexact", "st_plan_set_variant", "st_plan_autotune", "st_plan_autotune_report", "st_plan_sync",
           "st_plan_set_dist", "st_plan_set_loopback_slabs", "st_plan_ghost_planes", "st_plan_local_slab",
           "st_plan_get_info", "st_plan_last_launches", "st_blocking_model", "st_fig3_step",
           "st_nccl_unique_id", "st_slab_range", "st_slab_schedule"]


def lib() -> ctypes.CDLL:
    """Load libst35d.so (raises if it was not built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(LIB_PATH)
    P, I, D = ctypes.c_void_p, ctypes.c_int, ctypes.c_double
    sig = {
        "st_plan_create": ([I, I, I, I, I], P),
        "st7_run": ([P, P, P, D, D, I], I),
        "st27_run": ([P, P, P, D, D, D, D, I], I),
        "st13_run": ([P, P, P, D, D, D, I], I),
        "lbm_d3q19_run": ([P, P, P, D, I, P], I),
        "st_destroy": ([P], None),
        "st_last_error": ([], ctypes.c_char_p),
        "st_last_status": ([], I),
        "st_plan_set_stream": ([P, P], I),
        "st_plan_set_lbm_lid": ([P, D, D, D], I),
        "st_plan_set_option": ([P, I, I], I),
        "st_plan_set_bitexact": ([P, I], I),
        "st_plan_set_variant": ([P, I], I),
        "st_plan_autotune": ([P, P, P, I, ctypes.POINTER(I), ctypes.POINTER(ctypes.c_float)], I),
        "st_plan_autotune_report": ([P, P, P, I, ctypes.POINTER(st_autotune_report)], I),
        "st_plan_sync": ([P], I),
        "st_plan_set_dist": ([P, P, I, I], I),
        "st_plan_set_loopback_slabs": ([P, I], I),
        "st_plan_ghost_planes": ([P], I),
        "st_plan_local_slab": ([P, ctypes.POINTER(I), ctypes.POINTER(I)], I),
        "st_plan_get_info": ([P, I, ctypes.POINTER(st_plan_info)], I),
        "st_plan_last_launches": ([P], I),
        "st_blocking_model": ([D, D, I, D, D, I, I, ctypes.POINTER(st_blocking)], I),
        "st_fig3_step": ([I, I, I, I, ctypes.POINTER(I), ctypes.POINTER(I)], I),
        "st_nccl_unique_id": ([P], I),
        "st_slab_range": ([I, I, I, ctypes.POINTER(I), ctypes.POINTER(I)], I),
        "st_slab_schedule": ([I, I, I, I, I, I, ctypes.POINTER(st_slab_step), I], I),
    }
    for name, (args, res) in sig.items():
        if os.environ.get("ST35D_LIB") and not hasattr(L, name):   # A/B build of an older ABI
            continue
        fn = getattr(L, name)
        fn.argtypes = args
        fn.restype = res
    _lib = L
    return L


def st_last_error() -> str:
    return lib().st_last_error().decode()


def _check(rc: int) -> int:
    if rc < 0:
        raise StError(rc, st_last_error())
    return rc


def _ptr(buf) -> int:
    """device or host address of a torch tensor / numpy array / int."""
    if buf is None:
        return 0
    if isinstance(buf, int):
        return buf
    if hasattr(buf, "data_ptr"):
        if not buf.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return buf.data_ptr()
    if hasattr(buf, "ctypes"):
        if not buf.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return buf.ctypes.data
    raise TypeError(type(buf))


def st_plan_create(nx: int, ny: int, nz: int, dtype: int, dim_T: int) -> int:
    h = lib().st_plan_create(nx, ny, nz, dtype, dim_T)
    if not h:
        raise StError(lib().st_last_status() or ST_EINVAL, st_last_error())
    return h


def st7_run(plan: int, inp, out, alpha: float, beta: float, T: int) -> int:
    return _check(lib().st7_run(plan, _ptr(inp), _ptr(out), alpha, beta, T))


def st13_run(plan: int, inp, out, alpha: float, beta: float, gamma: float, T: int) -> int:
    return _check(lib().st13_run(plan, _ptr(inp), _ptr(out), alpha, beta, gamma, T))


def st27_run(plan: int, inp, out, alpha: float, beta: float, gamma: float, delta: float, T: int) -> int:
    return _check(lib().st27_run(plan, _ptr(inp), _ptr(out), alpha, beta, gamma, delta, T))


def lbm_d3q19_run(plan: int, f_src, f_dst, omega: float, T: int, flags) -> int:
    return _check(lib().lbm_d3q19_run(plan, _ptr(f_src), _ptr(f_dst), omega, T, _ptr(flags)))


def st_destroy(plan: int) -> None:
    if plan:
        lib().st_destroy(plan)


def st_plan_set_stream(plan: int, stream) -> int:
    s = stream if isinstance(stream, int) else getattr(stream, "cuda_stream", 0)
    return _check(lib().st_plan_set_stream(plan, s))


def st_plan_set_lbm_lid(plan: int, ux: float, uy: float, uz: float) -> int:
    return _check(lib().st_plan_set_lbm_lid(plan, ux, uy, uz))


def st_plan_set_option(plan: int, option: int, value: int) -> int:
    """ST_OPT_* tuning / test selections (include/st35d.h); results do not depend on them."""
    return _check(lib().st_plan_set_option(plan, int(option), int(value)))


def st_plan_set_bitexact(plan: int, on: bool) -> int:
    return _check(lib().st_plan_set_bitexact(plan, 1 if on else 0))


ST_VARIANT_35D, ST_VARIANT_NAIVE = 0, 1


def st_plan_set_variant(plan: int, variant: int) -> int:
    """ST_VARIANT_NAIVE: the no-blocking ablation baseline (include/st35d.h)."""
    return _check(lib().st_plan_set_variant(plan, int(variant)))


def st_plan_autotune(plan: int, a, b, T_probe: int):
    """returns (chosen dim_T, eq. (3) eta seed, {dim_T: ms for T_probe steps})."""
    eta = ctypes.c_int()
    ms = (ctypes.c_float * 16)()
    d = _check(lib().st_plan_autotune(plan, _ptr(a), _ptr(b), T_probe, ctypes.byref(eta), ms))
    return d, eta.value, {k + 1: ms[k] for k in range(16) if ms[k] > 0}


def st_plan_autotune_report(plan: int, a, b, T_probe: int) -> dict:
    """model-seeded depth search (include/st35d.h); returns the report as a dict."""
    r = st_autotune_report()
    _check(lib().st_plan_autotune_report(plan, _ptr(a), _ptr(b), T_probe, ctypes.byref(r)))
    out = {k: getattr(r, k) for k, _ in st_autotune_report._fields_}
    for k in ("tested", "ms", "capacity", "tile_side", "kappa"):
        out[k] = list(out[k])
    out["ms"] = {d + 1: round(v, 4) for d, v in enumerate(out["ms"]) if v > 0}
    return out


def st_plan_sync(plan: int) -> int:
    return _check(lib().st_plan_sync(plan))


def st_plan_set_dist(plan: int, unique_id: bytes, rank: int, nranks: int) -> int:
    buf = ctypes.create_string_buffer(bytes(unique_id), 128)
    return _check(lib().st_plan_set_dist(plan, ctypes.addressof(buf), rank, nranks))


def st_plan_set_loopback_slabs(plan: int, nslabs: int) -> int:
    return _check(lib().st_plan_set_loopback_slabs(plan, nslabs))


def st_plan_ghost_planes(plan: int) -> int:
    return _check(lib().st_plan_ghost_planes(plan))


def st_plan_local_slab(plan: int):
    z0, n = ctypes.c_int(), ctypes.c_int()
    _check(lib().st_plan_local_slab(plan, ctypes.byref(z0), ctypes.byref(n)))
    return z0.value, n.value


def st_plan_get_info(plan: int, lbm: bool = False) -> dict:
    info = st_plan_info()
    _check(lib().st_plan_get_info(plan, 1 if lbm else 0, ctypes.byref(info)))
    return {k: getattr(info, k) for k, _ in st_plan_info._fields_}


def st_plan_last_launches(plan: int) -> int:
    return _check(lib().st_plan_last_launches(plan))


def st_blocking_model(C_bytes: float, E_bytes: float, R: int, gamma: float, Gamma: float,
                      dim_T: int = 0, dim: int = 0) -> dict:
    out = st_blocking()
    _check(lib().st_blocking_model(C_bytes, E_bytes, R, gamma, Gamma, dim_T, dim, ctypes.byref(out)))
    return {k: getattr(out, k) for k, _ in st_blocking._fields_}


def st_fig3_step(R: int, dim_T: int, rnd: int, level: int):
    z, s = ctypes.c_int(), ctypes.c_int()
    step = _check(lib().st_fig3_step(R, dim_T, rnd, level, ctypes.byref(z), ctypes.byref(s)))
    return step, z.value, s.value


def st_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().st_nccl_unique_id(ctypes.addressof(buf)))
    return buf.raw


def st_slab_range(nz: int, nranks: int, rank: int):
    z0, n = ctypes.c_int(), ctypes.c_int()
    _check(lib().st_slab_range(nz, nranks, rank, ctypes.byref(z0), ctypes.byref(n)))
    return z0.value, n.value


def st_slab_schedule(nz: int, nranks: int, rank: int, dim_T: int, T: int, overlap: bool = True) -> list:
    """the Z-slab step list a rank executes (include/st35d.h), as dicts."""
    n = _check(lib().st_slab_schedule(nz, nranks, rank, dim_T, T, 1 if overlap else 0, None, 0))
    buf = (st_slab_step * max(n, 1))()
    _check(lib().st_slab_schedule(nz, nranks, rank, dim_T, T, 1 if overlap else 0, buf, n))
    return [{"kind": s.kind, "sweep": s.sweep, "depth": s.depth, "src": s.src, "z_begin": s.z_begin,
             "z_end": s.z_end, "async": s.async_, "grid_cap": s.grid_cap} for s in buf[:n]]


def dtype_code(dtype) -> int:
    name = str(dtype)
    if "float32" in name:
        return ST_F32
    if "float64" in name:
        return ST_F64
    raise ValueError(f"unsupported dtype {dtype}")


def _buf_info(buf):
    """(is_device, element size, dtype code or None, numel) of a tensor / array."""
    if hasattr(buf, "data_ptr"):   # torch tensor
        dev = buf.device.type == "cuda"
        name = str(buf.dtype)
        return dev, buf.element_size(), name, buf.numel()
    if hasattr(buf, "ctypes"):     # numpy array
        return False, buf.itemsize, str(buf.dtype), buf.size
    return None


class Plan:
    """RAII wrapper: ``with Plan(nx, ny, nz, dtype, dim_T) as p: p.st7(a, b, ...)``.

    The methods check each tensor / array against the plan (device or host,
    dtype, element count) before calling the C ABI, which only sees pointers
    and could not detect a short or mistyped buffer (ValueError on mismatch).
    Raw integer addresses are passed through unchecked."""

    def __init__(self, nx: int, ny: int, nz: int, dtype, dim_T: int):
        self.dtype = dtype if isinstance(dtype, int) else dtype_code(dtype)
        self.h = st_plan_create(nx, ny, nz, self.dtype, dim_T)
        self.shape = (nz, ny, nx)
        self._nzb = nz

    def _local_cells(self) -> int:
        nz, ny, nx = self.shape
        return nx * ny * self._nzb

    def _check_bufs(self, bufs, ncomp: int, what: str) -> None:
        want = "float32" if self.dtype == ST_F32 else "float64"
        need = ncomp * self._local_cells()
        kinds = set()
        for b in bufs:
            info = _buf_info(b)
            if info is None:
                continue
            dev, _, name, n = info
            kinds.add(dev)
            if want not in name:
                raise ValueError(f"{what}: buffer dtype {name} does not match the plan ({want})")
            if n != need:
                raise ValueError(f"{what}: buffer has {n} elements, the plan needs {need}")
        if len(kinds) > 1:
            raise ValueError(f"{what}: buffers must all be on the device or all on the host")

    def _check_flags(self, flags, ref) -> None:
        info = _buf_info(flags)
        if info is None:
            return
        dev, esz, name, n = info
        if "uint8" not in name:
            raise ValueError(f"flags must be uint8, got {name}")
        if n != self._local_cells():
            raise ValueError(f"flags have {n} elements, the plan needs {self._local_cells()}")
        r = _buf_info(ref)
        if r is not None and r[0] != dev:
            raise ValueError("flags and populations must both be on the device or both on the host")

    def st7(self, inp, out, alpha: float, beta: float, T: int) -> None:
        self._check_bufs((inp, out), 1, "st7")
        st7_run(self.h, inp, out, alpha, beta, T)

    def st13(self, inp, out, alpha: float, beta: float, gamma: float, T: int) -> None:
        self._check_bufs((inp, out), 1, "st13")
        st13_run(self.h, inp, out, alpha, beta, gamma, T)

    def st27(self, inp, out, alpha: float, beta: float, gamma: float, delta: float, T: int) -> None:
        self._check_bufs((inp, out), 1, "st27")
        st27_run(self.h, inp, out, alpha, beta, gamma, delta, T)

    def lbm(self, f_src, f_dst, omega: float, T: int, flags) -> None:
        self._check_bufs((f_src, f_dst), 19, "lbm")
        self._check_flags(flags, f_src)
        lbm_d3q19_run(self.h, f_src, f_dst, omega, T, flags)

    def set_option(self, option: int, value: int) -> None:
        st_plan_set_option(self.h, option, value)

    def set_dist(self, unique_id: bytes, rank: int, nranks: int) -> None:
        st_plan_set_dist(self.h, unique_id, rank, nranks)
        self._nzb = st_plan_local_slab(self.h)[1] + 2 * st_plan_ghost_planes(self.h)   # slab + ghosts

    def set_stream(self, stream) -> None:
        st_plan_set_stream(self.h, stream)

    def autotune(self, a, b, T_probe: int):
        return st_plan_autotune(self.h, a, b, T_probe)

    def autotune_report(self, a, b, T_probe: int) -> dict:
        return st_plan_autotune_report(self.h, a, b, T_probe)

    def set_variant(self, variant: int) -> None:
        st_plan_set_variant(self.h, variant)

    def set_bitexact(self, on: bool) -> None:
        st_plan_set_bitexact(self.h, on)

    def set_lid(self, ux: float, uy: float, uz: float) -> None:
        st_plan_set_lbm_lid(self.h, ux, uy, uz)

    def sync(self) -> None:
        st_plan_sync(self.h)

    def info(self, lbm: bool = False) -> dict:
        return st_plan_get_info(self.h, lbm)

    def last_launches(self) -> int:
        return st_plan_last_launches(self.h)

    def close(self) -> None:
        if self.h:
            st_destroy(self.h)
            self.h = 0

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
