"""Build libst35d.so (the C-ABI library) in-tree with nvcc for sm_100a.

Objects are compiled in parallel; st7_inst.cu is compiled once per
(dtype, mode) with -D switches.  Re-running only rebuilds stale objects.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
# A/B tuning builds: ST_AB=name builds build/ab/<name>/libst35d.so with the
# extra -D flags in ST_AB_DEFS (load it with ST35D_LIB=...); the default build
# is the in-tree product library.
_AB = os.environ.get("ST_AB")
BUILD = os.path.join(ROOT, "build", "ab", _AB, "obj") if _AB else os.path.join(ROOT, "build", "obj")
LIB = os.path.join(ROOT, "build", "ab", _AB, "libst35d.so") if _AB else os.path.join(PKG, "libst35d.so")
_AB_DEFS = os.environ.get("ST_AB_DEFS", "").split() if _AB else []
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nccl_include():
    try:
        import importlib.util
        spec = importlib.util.find_spec("nvidia")
        if spec and spec.submodule_search_locations:
            for loc in spec.submodule_search_locations:
                inc = os.path.join(loc, "nccl", "include")
                if os.path.exists(os.path.join(inc, "nccl.h")):
                    return inc
    except Exception:
        pass
    return None


_NCCL_INC = _nccl_include()
COMMON = ARCH + ["-O3", "-lineinfo", "-std=c++20", "--expt-relaxed-constexpr", "-Xcompiler", "-fPIC",
                 "-Xcompiler", "-ffp-contract=off", "-I", os.path.join(ROOT, "include")] + \
    (["-DST_HAVE_NCCL=1", "-I", _NCCL_INC] if _NCCL_INC else ["-DST_HAVE_NCCL=0"]) + _AB_DEFS

UNITS = [
    ("api.cu", "api.o", []),
    ("lbm_inst.cu", "lbm_inst.o", []),
    ("lbm_tma.cu", "lbm_tma.o", []),
    ("naive.cu", "naive.o", []),
    ("st27.cu", "st27.o", []),
    ("st13_inst.cu", "st13_inst.o", []),
    ("st27t_inst.cu", "st27t_inst.o", []),
    ("model.cpp", "model.o", []),
] + [
    ("st7_inst.cu", f"st7_{tn}_{mode}.o", [f"-DST_T={t}", f"-DST_TNAME={tn}", f"-DST_EXACT={ex}"])
    for t, tn in (("float", "f32"), ("double", "f64"))
    for mode, ex in (("fast", 0), ("exact", 1))
]


def _deps():
    return sorted(glob.glob(os.path.join(CSRC, "*")) + glob.glob(os.path.join(ROOT, "include", "*.h")))


def _unit_deps(obj: str) -> list[str]:
    """headers the object was compiled from (nvcc -MD), else every source file"""
    dep = obj + ".d"
    if not os.path.exists(dep):
        return _deps()
    txt = open(dep).read().replace("\\\n", " ")
    files = [f for f in txt.split(":", 1)[-1].split() if f.startswith(ROOT)]
    return files + [os.path.abspath(__file__)] if files else _deps()


def _stale(obj: str, src: str) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(not os.path.exists(d) or os.path.getmtime(d) > t for d in _unit_deps(obj))


def _compile(src, obj, extra, verbose):
    md = ["-MD", "-MF", obj + ".d"]
    cmd = [NVCC, *COMMON, *extra, *md, "-c", os.path.join(CSRC, src), "-o", obj]
    if src.endswith(".cpp"):
        cmd = [NVCC, *COMMON, *extra, *md, "-x", "cu", "-c", os.path.join(CSRC, src), "-o", obj]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        cmd.insert(1, "-Xptxas=-warn-spills")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr[-6000:]}")
    return r.stderr


def build(force: bool = False, verbose: bool = False, jobs: int | None = None) -> str:
    os.makedirs(BUILD, exist_ok=True)
    todo = []
    objs = []
    only = os.environ.get("ST_AB_ONLY", "").split(",") if _AB else [""]
    for src, obj, extra in UNITS:
        o = os.path.join(BUILD, obj)
        if _AB and only != [""] and obj[:-2] not in only:   # reuse the product build's object
            o = os.path.join(ROOT, "build", "obj", obj)
            objs.append(o)
            continue
        objs.append(o)
        if force or _stale(o, src):
            todo.append((src, o, extra))
    logs = {}
    if todo:
        with cf.ThreadPoolExecutor(max_workers=jobs or min(len(todo), os.cpu_count() or 4)) as ex:
            futs = {ex.submit(_compile, s, o, e, verbose): s for s, o, e in todo}
            for f in cf.as_completed(futs):
                logs[futs[f]] = f.result()
    stale_lib = not os.path.exists(LIB) or any(os.path.getmtime(o) > os.path.getmtime(LIB) for o in objs)
    if todo or stale_lib:
        tmp = LIB + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-Xcompiler", "-fPIC", "-ldl"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr[-4000:]}")
        os.replace(tmp, LIB)
    if verbose:
        for k, v in logs.items():
            sys.stderr.write(f"== {k}\n{v}\n")
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
