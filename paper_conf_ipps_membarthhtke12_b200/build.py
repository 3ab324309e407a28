"""Build liblop.so (the C-ABI library + sm_100a kernels) in-tree with nvcc.

    python paper_conf_ipps_membarthhtke12_b200/build.py [--force] [--verbose]

Every translation unit is compiled for sm_100a only
(-gencode arch=compute_100a,code=sm_100a), with -lineinfo so ncu's source
page maps to csrc/, and linked with the static CUDA runtime so the library
loads without a torch-matched libcudart.  `-Xptxas -v` register/spill
reports are written to build/ptxas_<unit>.log.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
BUILD = os.path.join(PKG, "build")
LIB = os.path.join(PKG, "liblop.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC)
                  if f.endswith((".cu", ".cpp")))


def headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    return hs + [os.path.join(INCLUDE, "lop.h")]


def deps(src: str, seen=None) -> set:
    """The in-tree headers `src` includes, transitively (#include "...")."""
    import re
    seen = set() if seen is None else seen
    with open(src) as f:
        for name in re.findall(r'^\s*#\s*include\s+"([^"]+)"', f.read(), re.M):
            for d in (CSRC, INCLUDE):
                h = os.path.join(d, name)
                if os.path.exists(h) and h not in seen:
                    seen.add(h)
                    deps(h, seen)
                    break
    return seen


def _compile(src: str, force: bool, verbose: bool) -> str:
    unit = os.path.splitext(os.path.basename(src))[0]
    obj = os.path.join(BUILD, unit + ".o")
    newest_dep = max([os.path.getmtime(src)] + [os.path.getmtime(h) for h in deps(src)])
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= newest_dep:
        return obj
    cmd = [nvcc(), *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC",
           "-I", INCLUDE, "-I", CSRC, "-c", src, "-o", obj]
    if src.endswith(".cu"):
        cmd[1:1] = ["-Xptxas", "-v", "--expt-relaxed-constexpr"]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if src.endswith(".cu"):
        with open(os.path.join(BUILD, "ptxas_%s.log" % unit), "w") as f:
            f.write(res.stderr)
    if res.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, " ".join(cmd), res.stderr))
    if verbose:
        print(" ".join(cmd))
    return obj


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    srcs = sources()
    with cf.ThreadPoolExecutor(max_workers=min(8, len(srcs))) as ex:
        objs = list(ex.map(lambda s: _compile(s, force, verbose), srcs))
    if force or not os.path.exists(LIB) or max(map(os.path.getmtime, objs)) > os.path.getmtime(LIB):
        tmp = LIB + ".tmp%d" % os.getpid()
        cmd = [nvcc(), *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            raise RuntimeError("link failed:\n%s\n%s" % (" ".join(cmd), res.stderr))
        os.replace(tmp, LIB)
    return LIB


EXAMPLE_SRC = os.path.join(ROOT, "examples", "bilateral_c.c")
EXAMPLE_BIN = os.path.join(ROOT, "examples", "bilateral_c")


def build_example(force: bool = False) -> str:
    """Plain-C program against include/lop.h + liblop.so (the ABI without Python)."""
    lib = build(force=force)
    if not force and os.path.exists(EXAMPLE_BIN) and \
            os.path.getmtime(EXAMPLE_BIN) >= max(os.path.getmtime(EXAMPLE_SRC),
                                                 os.path.getmtime(lib)):
        return EXAMPLE_BIN
    cmd = [nvcc(), *ARCH, "-O2", "-x", "cu", "-I", INCLUDE, EXAMPLE_SRC, "-o", EXAMPLE_BIN,
           "-L", PKG, "-llop", "-Xlinker", "-rpath=$ORIGIN/../" + os.path.basename(PKG)]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError("example build failed:\n%s\n%s" % (" ".join(cmd), res.stderr))
    return EXAMPLE_BIN


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("--verbose", action="store_true")
    a = ap.parse_args(argv)
    print(build(force=a.force, verbose=a.verbose))
    print(build_example(force=a.force))


if __name__ == "__main__":
    sys.exit(main())
