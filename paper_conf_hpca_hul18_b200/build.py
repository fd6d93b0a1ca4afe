"""Build libnfc.so (the C-ABI library) in-tree with nvcc for sm_100a.

Each translation unit is compiled to an object in parallel (the kernel
instantiations are split across sfc_inst_*.cu), then linked into one shared
library."""
from __future__ import annotations

import glob
import os
import subprocess
import sys
import tempfile
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libnfc.so")
ROOT = os.path.dirname(HERE)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    s = ["capi.cu", "sfc_kernel.cu", "unfused.cu", "builders.cpp", "debug_host.cpp", "planner.cpp", "parallel.cu", "dpi_stream.cu", "regex.cpp", "comm.cu", "peaks.cu"]
    s += sorted(os.path.basename(p) for p in glob.glob(os.path.join(CSRC, "sfc_inst_*.cu")))
    return s


def headers():
    return [os.path.join(CSRC, h) for h in ("nfc_internal.h", "sfc_kernel.cuh")] + \
           [os.path.join(ROOT, "include", f) for f in ("nfc.h", "nfc_debug.h")]


def _stale(lib) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = [os.path.join(CSRC, s) for s in sources()] + headers() + [os.path.abspath(__file__)]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, defines=(), out=None) -> str:
    """Build libnfc.so; `defines`/`out` build an experimental variant elsewhere."""
    target = out or LIB
    if not force and not _stale(target):
        return target
    common = [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
              "-I", os.path.join(ROOT, "include"), *[f"-D{d}" for d in defines]]
    tmp = tempfile.mkdtemp(prefix="nfc_build_")

    def compile_one(src):
        obj = os.path.join(tmp, src + ".o")
        cmd = [NVCC, *common, "-Xptxas", "-v" if verbose else "-O3", "-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        return src, obj, r

    with ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 4)) as ex:
        results = list(ex.map(compile_one, sources()))
    for src, _, r in results:
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed on {src}")
        if verbose:
            sys.stderr.write(f"== {src}\n" + r.stderr)
    objs = [o for _, o, _ in results]
    link = [NVCC, *ARCH, "-shared", "-o", target + ".tmp", *objs, "-ldl"]
    r = subprocess.run(link, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc link of libnfc.so failed")
    os.replace(target + ".tmp", target)
    for o in objs:
        os.remove(o)
    os.rmdir(tmp)
    return target


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
