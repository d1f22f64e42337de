"""Build the CUDA C-ABI library in-tree (sm_100a only) with nvcc.

The .so lands next to this file so it travels with the repo snapshot to the
GPU box (it is git-ignored, not gpurun-ignored).
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libga.so")
SOURCES = ["ga_host.cu", "ga_bench.cu", "ga_rcu.cu"]
DEPS = SOURCES + ["ga_device_impl.cuh", "ga_internal.h"]
HEADERS = ["ga.h", "ga_bench.h", "ga_device.cuh", "ga_rcu.h"]

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
              "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-warn-spills"]


def _stale(lib: str = LIB) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    srcs = [os.path.join(CSRC, f) for f in DEPS] + [os.path.join(INCLUDE, f) for f in HEADERS]
    return any(os.path.getmtime(s) > t for s in srcs)


# Build variants the tests load through GA_LIB (each a complete libga.so):
#   nspan0 -- GA_NSPAN=0, the paper's routing (every size above the bins on
#             TBuddy), run by the parity suite (tests/test_gpu_variants.py).
VARIANTS = {"nspan0": ("GA_NSPAN=0",)}


def variant_path(name: str) -> str:
    return os.path.join(PKG, f"libga_{name}.so")


def build_variants(force: bool = False) -> dict:
    """Compile every VARIANTS entry next to libga.so (if missing or stale)."""
    out = {}
    for name, defines in VARIANTS.items():
        path = variant_path(name)
        if force or not os.path.exists(path) or _stale(path):
            build(defines=defines, out=path)
        out[name] = path
    return out


def build_all(force: bool = False) -> None:
    """libga.so and every variant, concurrently."""
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(2) as ex:
        a = ex.submit(build, force)
        b = ex.submit(build_variants, force)
        a.result()
        b.result()


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Compile libga.so if missing or older than its sources; returns its path.
    `defines` / `out` build a tuning variant (e.g. ("GA_LVL_HINT=1",)) elsewhere."""
    target = out or LIB
    if not force and not defines and out is None and not _stale():
        return LIB
    nvcc = os.environ.get("NVCC", "nvcc")
    # one nvcc per translation unit, in parallel (each TU carries its own copy
    # of the allocator's device code), then one shared-library link
    flags = [f for f in NVCC_FLAGS if f != "-shared"]
    common = [*flags, *[f"-D{d}" for d in defines], "-I", INCLUDE, "-I", CSRC]
    if verbose:
        common = ["-Xptxas", "-v", *common]
    objs = [f"{target}.{os.path.splitext(f)[0]}.o" for f in SOURCES]

    def compile_one(src_obj):
        src, obj = src_obj
        return subprocess.run([nvcc, *common, "-c", os.path.join(CSRC, src), "-o", obj], capture_output=True, text=True)

    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(len(SOURCES)) as ex:
        results = list(ex.map(compile_one, zip(SOURCES, objs)))
    for r in results:
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed building libga.so")
        if verbose:
            sys.stderr.write(r.stderr)
    r = subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-Xcompiler", "-fPIC",
                        *objs, "-o", target + ".tmp"], capture_output=True, text=True)
    for o in objs:
        if os.path.exists(o):
            os.remove(o)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed linking libga.so")
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    build(force=True, verbose="-v" in sys.argv)
    print(LIB)
    for path in build_variants(force=True).values():
        print(path)
