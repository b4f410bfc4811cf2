"""Build libifl.so (sm_100a) in-tree with nvcc.

    python -m paper_conf_ppopp_henriksenteo19_b200.build [--force] [-j N]

Every .cu / .cpp under csrc/ is compiled to an object with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` and linked into
``paper_conf_ppopp_henriksenteo19_b200/libifl.so`` (static cudart).  Objects
are rebuilt only when their source or a header is newer.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
# IFL_BUILD_TAG builds an experiment variant side by side (build_obj_<tag>,
# libifl_<tag>.so; load it with IFL_LIB_PATH) -- tools only, never the product
_TAG = os.environ.get("IFL_BUILD_TAG", "")
OBJ = os.path.join(PKG, "build_obj" + (f"_{_TAG}" if _TAG else ""))
LIB = os.path.join(PKG, "libifl" + (f"_{_TAG}" if _TAG else "") + ".so")
NVCC = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-I" + CSRC, "-I" + os.path.join(ROOT, "include")]
CUFLAGS = ARCH + COMMON + ["-lineinfo", "--expt-relaxed-constexpr", "-Xptxas", "-warn-spills"]
# experiment builds only: extra -D flags for a tagged variant (IFL_BUILD_EXTRA="-DX=1 ...")
if _TAG:
    CUFLAGS = CUFLAGS + os.environ.get("IFL_BUILD_EXTRA", "").split()


def _headers():
    return glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h")) + [
        os.path.join(ROOT, "include", "ifl.h")]


def _stale(src: str, obj: str, hdr_mtime: float) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return t < os.path.getmtime(src) or t < hdr_mtime


def _compile(src: str, obj: str, extra):
    cmd = [NVCC] + (CUFLAGS if src.endswith(".cu") else ARCH + COMMON) + list(extra) + ["-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {os.path.basename(src)}:\n{r.stderr}")
    return src, r.stderr


def build(force: bool = False, jobs: int | None = None, verbose: bool = False, extra=()) -> str:
    os.makedirs(OBJ, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))
    hdr = max(os.path.getmtime(h) for h in _headers())
    todo = []
    objs = []
    only = os.environ.get("IFL_BUILD_ONLY", "").split() if _TAG else []  # experiment builds: recompile these only
    main_obj = os.path.join(PKG, "build_obj")
    for s in srcs:
        o = os.path.join(OBJ, os.path.basename(s) + ".o")
        if only and os.path.basename(s) not in only:
            o = os.path.join(main_obj, os.path.basename(s) + ".o")  # the product build's object
            objs.append(o)
            continue
        objs.append(o)
        if force or _stale(s, o, hdr):
            todo.append((s, o))
    if todo:
        jobs = jobs or min(len(todo), os.cpu_count() or 4)
        with cf.ThreadPoolExecutor(jobs) as ex:
            for src, err in ex.map(lambda so: _compile(so[0], so[1], extra), todo):
                if verbose and err.strip():
                    print(f"[{os.path.basename(src)}]\n{err}", file=sys.stderr)
    if todo or not os.path.exists(LIB) or any(os.path.getmtime(o) > os.path.getmtime(LIB) for o in objs):
        cmd = [NVCC] + ARCH + ["-shared", "-o", LIB] + objs + ["-lcuda"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
    return LIB


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=None)
    ap.add_argument("-v", action="store_true")
    a = ap.parse_args()
    print(build(a.force, a.j, a.v))
