"""Build libooo.so (the C-ABI library) in-tree with nvcc for sm_100a.

    python -m paper_conf_eurosys_ohlks22_b200.build [--force]

Objects are compiled in parallel; the shared library links the CUDA runtime
statically and loads NCCL at run time (dlopen), so it loads on hosts without
a GPU or NCCL (host-only entry points work there).
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIBDIR = os.path.join(PKG, "lib")
LIB = os.path.join(LIBDIR, "libooo.so")
OBJDIR = os.path.join(PKG, "build_obj")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["engine.cu", "skinny.cu", "gemm_simt.cu", "ew.cu", "ooo_api.cpp", "nccl_dyn.cpp", "planner.cpp", "regions.cpp", "comm_order.cpp", "pipeline.cpp"]


def _nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _nccl_include() -> str:
    try:
        import nvidia.nccl  # noqa: F401  (torch's bundled NCCL: the copy loaded at run time)
        base = os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0]
        inc = os.path.join(base, "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    except Exception:
        pass
    if os.path.exists("/usr/include/nccl.h"):
        return "/usr/include"
    raise RuntimeError("nccl.h not found")


def _flags() -> list:
    return ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", "-I", INCLUDE,
                   "-I", _nccl_include(), "--expt-relaxed-constexpr"]


def _digest() -> str:
    h = hashlib.sha256()
    for name in sorted(os.listdir(CSRC)):
        with open(os.path.join(CSRC, name), "rb") as f:
            h.update(name.encode() + f.read())
    with open(os.path.join(INCLUDE, "ooo.h"), "rb") as f:
        h.update(f.read())
    h.update(" ".join(_flags()).encode())
    return h.hexdigest()


def build(force: bool = False, verbose: bool = True, trace: bool = False, variant: str = "",
          defines: tuple = ()) -> str:
    """trace=True builds the debug variant lib/libooo_trace.so (-DOOO_TRACE:
    per-task timestamps in the engine, tools/engine_trace.py); `variant` +
    `defines` build tuning variants lib/libooo_<variant>.so."""
    name = ("libooo_trace" if trace else "libooo") + (f"_{variant}" if variant else "") + ".so"
    lib = os.path.join(LIBDIR, name)
    objdir = OBJDIR + ("_trace" if trace else "") + (f"_{variant}" if variant else "")
    os.makedirs(LIBDIR, exist_ok=True)
    os.makedirs(objdir, exist_ok=True)
    stamp = os.path.splitext(lib)[0] + ".sha256"
    dig = _digest() + ("-trace" if trace else "") + "".join(defines)
    if not force and os.path.exists(lib) and os.path.exists(stamp) and open(stamp).read() == dig:
        return lib
    nvcc = _nvcc()
    flags = _flags() + (["-DOOO_TRACE"] if trace else []) + [f"-D{d}" for d in defines]

    def compile_one(src):
        obj = os.path.join(objdir, src + ".o")
        cmd = [nvcc] + flags + ["-Xptxas", "-v"] * (src == "engine.cu" and verbose is None) + \
              ["-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
        return obj

    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        objs = list(ex.map(compile_one, SOURCES))
    tmp = lib + ".tmp"
    cmd = [nvcc] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs + ["-ldl", "-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, lib)
    with open(stamp, "w") as f:
        f.write(dig)
    if verbose:
        print(f"built {lib}", file=sys.stderr)
    return lib


if __name__ == "__main__":
    defs = tuple(a[2:] for a in sys.argv[1:] if a.startswith("-D"))
    var = next((a.split("=", 1)[1] for a in sys.argv[1:] if a.startswith("--variant=")), "")
    build(force="--force" in sys.argv, trace="--trace" in sys.argv, variant=var, defines=defs)
