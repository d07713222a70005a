"""Builds libgllm.so in-tree: nvcc for sm_100a (cross-compiles without a GPU).

    python -m paper_conf_sc_00090d00l25_b200.build [--force] [-v]

Every .cu is compiled with `-gencode arch=compute_100a,code=sm_100a -lineinfo
-O3`; .cpp files with the host compiler through nvcc.  Objects go to
build/obj/, the shared library to paper_conf_sc_00090d00l25_b200/libgllm.so.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INC = os.path.join(ROOT, "include")
OBJ = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(PKG, "libgllm.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
          f"-I{INC}", f"-I{CSRC}"]
CUFLAGS = ARCH + ["-lineinfo", "--expt-relaxed-constexpr", "-Xptxas", "-v" if os.environ.get("GLLM_PTXAS_V") else "-O3"]


def _deps_mtime():
    hs = glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(INC, "*.h"))
    return max((os.path.getmtime(h) for h in hs), default=0.0)


def _compile(src, force, verbose):
    base = os.path.splitext(os.path.basename(src))[0]
    ext = os.path.splitext(src)[1]
    obj = os.path.join(OBJ, base + (".cu.o" if ext == ".cu" else ".o"))
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), _deps_mtime()):
        return obj, None
    cmd = [NVCC] + COMMON + (CUFLAGS if ext == ".cu" else ["-x", "c++"]) + ["-c", src, "-o", obj]
    if verbose:
        print(" ".join(cmd), flush=True)
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        return obj, f"{' '.join(cmd)}\n{p.stdout}\n{p.stderr}"
    if verbose and p.stderr:
        print(p.stderr, flush=True)
    return obj, None


def build(force: bool = False, verbose: bool = False, variant: str = "") -> str:
    """variant "": libgllm.so.  variant "x": compiled with -DGLLM_VARIANT_X into libgllm_x.so
    (measurement builds selected at run time with GLLM_LIB=...)."""
    global OBJ, LIB, COMMON
    if variant:
        OBJ = os.path.join(ROOT, "build", "obj_" + variant)
        LIB = os.path.join(PKG, f"libgllm_{variant}.so")
        COMMON = COMMON + [f"-DGLLM_VARIANT_{variant.upper()}"]
    os.makedirs(OBJ, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))
    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        res = list(ex.map(lambda s: _compile(s, force, verbose), srcs))
    errs = [e for _, e in res if e]
    if errs:
        raise RuntimeError("nvcc failed:\n" + "\n".join(errs))
    objs = [o for o, _ in res]
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs):
        cmd = [NVCC] + ARCH + ["-shared", "-o", LIB] + objs + ["-ldl"]
        p = subprocess.run(cmd, capture_output=True, text=True)
        if p.returncode != 0:
            raise RuntimeError(f"link failed:\n{' '.join(cmd)}\n{p.stdout}\n{p.stderr}")
    return LIB


if __name__ == "__main__":
    var = next((a.split("=", 1)[1] for a in sys.argv if a.startswith("--variant=")), "")
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, variant=var))
