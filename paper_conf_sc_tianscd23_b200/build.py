"""Build libxs.so (the C-ABI library, include/xs.h) in-tree for sm_100a.

    python -m paper_conf_sc_tianscd23_b200.build [--force]

nvcc cross-compiles without a GPU; the .so lands next to this file so that
gpurun ships it to the B200 box with the repo snapshot.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libxs.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU_SOURCES = ["lookup.cu", "grid_build.cu", "xs_api.cu", "rs_lookup.cu"]
HEADERS = ["common.cuh", "radix_sort.cuh", "search.cuh", "xs_internal.h"]


def _deps():
    hs = [os.path.join(CSRC, h) for h in HEADERS]
    hs += [os.path.join(ROOT, "include", "xs.h"), os.path.join(ROOT, "include", "rs.h"),
           os.path.join(ROOT, "gen", "xs_gen.h"), os.path.join(ROOT, "gen", "rs_gen.h")]
    return hs


def _stale(out, srcs):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in srcs)


def _nvcc(src: str, verbose: bool) -> None:
    s = os.path.join(CSRC, src)
    o = os.path.join(BUILD, src + ".o")
    cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
           "-Xptxas", "-v", "-c", s, "-o", o]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if verbose or r.returncode:
        sys.stderr.write(r.stderr)
    if r.returncode:
        raise RuntimeError(f"nvcc failed for {src}")
    with open(o + ".ptxas.txt", "w") as f:
        f.write(r.stderr)


def build(force: bool = False, verbose: bool = False) -> str:
    from concurrent.futures import ThreadPoolExecutor
    os.makedirs(BUILD, exist_ok=True)
    objs = []
    deps = _deps()
    stale = []
    for src in CU_SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(BUILD, src + ".o")
        objs.append(o)
        if force or _stale(o, [s, *deps, __file__]):
            stale.append(src)
    # the translation units compile concurrently (lookup.cu dominates)
    with ThreadPoolExecutor(max_workers=max(1, len(stale))) as ex:
        for f in [ex.submit(_nvcc, src, verbose) for src in stale]:
            f.result()
    for gen in ("xs_gen", "rs_gen"):
        g = os.path.join(ROOT, "gen", gen + ".cpp")
        go = os.path.join(BUILD, gen + ".o")
        objs.append(go)
        if force or _stale(go, [g, os.path.join(ROOT, "gen", gen + ".h"),
                                os.path.join(ROOT, "gen", "xs_gen.h")]):
            subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-c", g, "-o", go])
    if force or _stale(LIB, objs):
        tmp = LIB + ".tmp"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lpthread"])
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
