"""Build the three native libraries in-tree (incremental, mtime-based).

* ``sfsgen/libsfsgen.so``   — seeded input generators (gcc, OpenMP)
* ``oracle/liboracle.so``   — CPU oracle (gcc -O2, no -march=native; test infrastructure)
* ``paper_conf_icppw_dhandhaniadpbl21_b200/libsfs.so`` — the product: CUDA kernels for sm_100a
  behind the C ABI of ``include/sfs.h`` (nvcc, ``-gencode arch=compute_100a,code=sm_100a``)

The oracle and the product are compiled from disjoint source trees with disjoint include paths.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.abspath(__file__))
PKG = os.path.join(ROOT, "paper_conf_icppw_dhandhaniadpbl21_b200")
CSRC = os.path.join(PKG, "csrc")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd):
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(" ".join(cmd) + "\n" + r.stdout + r.stderr)
        raise RuntimeError(f"build failed: {cmd[0]} … {cmd[-1]}")
    return r.stdout + r.stderr


def build_gen(force=False):
    src = [os.path.join(ROOT, "sfsgen", "gen.c"), os.path.join(ROOT, "sfsgen", "sfsgen.h")]
    out = os.path.join(ROOT, "sfsgen", "libsfsgen.so")
    if force or _stale(out, src):
        _run(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-fopenmp", src[0], "-o", out, "-lm"])
    return out


def build_gen_device(force=False):
    """sfsgen/libsfsgen_dev.so: the generators on the GPU (CUB sorts), bit-identical to gen.c."""
    src = [os.path.join(ROOT, "sfsgen", "gen_device.cu"), os.path.join(ROOT, "sfsgen", "sfsgen.h")]
    out = os.path.join(ROOT, "sfsgen", "libsfsgen_dev.so")
    if force or _stale(out, src):
        _run([NVCC, "-O3", "-std=c++17", "-shared", "-Xcompiler", "-fPIC,-ffp-contract=off", "-lineinfo"] + ARCH +
             ["-I", os.path.join(ROOT, "sfsgen"), src[0], "-o", out, "-cudart", "static"])
    return out


def build_oracle(force=False):
    src = [os.path.join(ROOT, "oracle", f) for f in ("oracle.c", "semisup.c", "oracle.h")]
    out = os.path.join(ROOT, "oracle", "liboracle.so")
    if force or _stale(out, src):
        _run(["gcc", "-O2", "-std=gnu11", "-ffp-contract=off", "-fPIC", "-shared", src[0], src[1], "-o", out, "-lm"])
    return out


def build_sfs(force=False, verbose=False, variant="", defines=()):
    cu = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    cpp = sorted(glob.glob(os.path.join(CSRC, "*.cpp")))
    hdr = sorted(glob.glob(os.path.join(CSRC, "*.cuh")) + glob.glob(os.path.join(CSRC, "*.h"))
                 + glob.glob(os.path.join(ROOT, "include", "*.h")))
    out = os.path.join(PKG, f"libsfs{variant}.so")
    if not (force or _stale(out, cu + cpp + hdr)):
        return out
    objdir = os.path.join(ROOT, "build", "obj" + variant)
    os.makedirs(objdir, exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC]
    common = ["-O3", "-std=c++17", "-Xcompiler", "-fPIC,-O3,-ffp-contract=off", "-lineinfo"] + inc + [f"-D{d}" for d in defines]

    def compile_one(src):
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        if force or _stale(obj, [src] + hdr):
            flags = ARCH + ["-Xptxas", "-v"] if src.endswith(".cu") else []
            log = _run([NVCC, "-c", src, "-o", obj] + common + flags + ["--expt-relaxed-constexpr"])
            if verbose and log:
                sys.stderr.write(log)
            with open(obj + ".log", "w") as fh:
                fh.write(log)
        return obj

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        objs = list(ex.map(compile_one, cu + cpp))
    _run([NVCC, "-shared"] + ARCH + ["-o", out] + objs + ["-cudart", "static", "-lpthread", "-ldl", "-lrt"])
    return out


def build_all(force=False):
    build_gen(force)
    build_gen_device(force)
    build_oracle(force)
    if glob.glob(os.path.join(CSRC, "*.cu")):
        build_sfs(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
    print("ok")
