"""Build the product library libtg.so (C ABI of include/tg.h) for sm_100a, in-tree.

nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3, one shared object with the
CUDA runtime linked statically; objects are rebuilt only when a source is newer.
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
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libtg.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-O2", "-Xptxas", "-v",
         f"-I{os.path.join(ROOT, 'include')}", f"-I{CSRC}", "--expt-relaxed-constexpr"]
# experiments only (tools/): extra -D flags build into their own object directory and always relink
EXTRA = os.environ.get("TG_NVCC_DEFS", "").split()
if EXTRA:
    BUILD = BUILD + "_" + "_".join(d.strip("-").replace("=", "") for d in EXTRA)


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cpp")) + glob.glob(os.path.join(CSRC, "*.cu"))
                  + glob.glob(os.path.join(CSRC, "kernels", "*.cu")))


def _headers_mtime():
    hs = (glob.glob(os.path.join(CSRC, "**", "*.h"), recursive=True)
          + glob.glob(os.path.join(CSRC, "**", "*.cuh"), recursive=True) + [os.path.join(ROOT, "include", "tg.h")])
    return max(os.path.getmtime(h) for h in hs)


def _compile(src: str, verbose: bool) -> str:
    rel = os.path.relpath(src, CSRC).replace(os.sep, "_")
    obj = os.path.join(BUILD, rel + ".o")
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(src), _headers_mtime()):
        return obj
    cmd = [NVCC, *ARCH, *FLAGS, *EXTRA, "-c", src, "-o", obj]
    if src.endswith(".cpp"):
        cmd = [NVCC, *ARCH, *FLAGS, *EXTRA, "-x", "cu", "-c", src, "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    if verbose:
        for line in (r.stdout + r.stderr).splitlines():
            if "registers" in line or "spill" in line or "warning" in line.lower():
                print(f"[{os.path.basename(src)}] {line.strip()}")
    return obj


def build(verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    srcs = sources()
    with ThreadPoolExecutor(max_workers=min(8, len(srcs))) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), srcs))
    stamp = LIB + ".flags"  # which -D flags the current libtg.so was linked from
    old = open(stamp).read() if os.path.exists(stamp) else ""
    if (EXTRA or old != " ".join(EXTRA) or not os.path.exists(LIB)
            or os.path.getmtime(LIB) < max(os.path.getmtime(o) for o in objs)):
        cmd = [NVCC, *ARCH, "-shared", "-o", LIB, *objs, "-lpthread"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stdout}\n{r.stderr}")
        with open(stamp, "w") as f:
            f.write(" ".join(EXTRA))
    return LIB


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv))
