"""Build the in-tree C-ABI library ``libpaella.so`` for sm_100a.

    python -m paper_conf_sosp_ngd023_b200.build

Host C++ (runtime, dispatcher, planner, policy) is compiled with g++; kernels with
nvcc ``-gencode arch=compute_100a,code=sm_100a -lineinfo``; everything is linked by
nvcc into one shared library with the static CUDA runtime.  Incremental: objects
are rebuilt when their source or any header is newer.

    python -m paper_conf_sosp_ngd023_b200.build --tsan

builds ``libpaella_tsan.so`` (host objects with ``-fsanitize=thread``, own build
directory) for the ThreadSanitizer run of the dispatcher (tools/sanitize.sh); load it
with ``PAELLA_LIB=<path>`` and ``LD_PRELOAD=<libtsan.so>``.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
OUT = os.path.join(HERE, "libpaella.so")
BUILD = os.path.join(HERE, "_build")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _newer(src, obj, headers):
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return os.path.getmtime(src) > t or any(os.path.getmtime(h) > t for h in headers)


def _run(cmd, verbose):
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError(f"build failed: {' '.join(cmd[:3])} ...")
    if verbose and (r.stdout or r.stderr):
        sys.stderr.write(r.stdout + r.stderr)


def build(verbose=False, ptxas_v=False, tsan=False):
    # A/B build variants: PAELLA_BUILD_VARIANT=<name> builds libpaella_<name>.so in its own
    # directory with the extra -D flags of PAELLA_DEFINES (load it with PAELLA_LIB)
    variant = os.environ.get("PAELLA_BUILD_VARIANT", "") or ("tsan" if tsan else "")
    defines = os.environ.get("PAELLA_DEFINES", "").split() if variant else []
    build_dir = BUILD + ("_" + variant if variant else "")
    out = os.path.join(HERE, f"libpaella_{variant}.so") if variant else OUT
    san = ["-fsanitize=thread"] if tsan else []
    os.makedirs(build_dir, exist_ok=True)
    headers = glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "paella.h")]
    objs = []
    inc = ["-I", CSRC, "-I", os.path.join(ROOT, "include"), "-I", os.path.join(CUDA, "include")]
    for src in sorted(glob.glob(os.path.join(CSRC, "*.cpp"))):
        obj = os.path.join(build_dir, os.path.basename(src) + ".o")
        objs.append(obj)
        if _newer(src, obj, headers):
            _run(["g++", "-O2", "-g", "-fPIC", *san, *defines, "-std=c++17", "-Wall", "-Wno-unused-function",
                  "-Wno-sign-compare", *inc, "-c", src, "-o", obj], verbose)
    for src in sorted(glob.glob(os.path.join(CSRC, "*.cu"))):
        obj = os.path.join(build_dir, os.path.basename(src) + ".o")
        objs.append(obj)
        if _newer(src, obj, headers):
            extra = ["-Xptxas", "-v"] if ptxas_v else []
            _run([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", *inc, *extra, *defines,
                  "-c", src, "-o", obj], verbose or ptxas_v)
    if not os.path.exists(out) or any(os.path.getmtime(o) > os.path.getmtime(out) for o in objs):
        tmp = out + ".tmp"
        _run([NVCC, *ARCH, "-shared", "-o", tmp, *objs, *(["-Xcompiler", "-fsanitize=thread"] if tsan else []),
              "-lpthread", "-lrt", "-ldl"], verbose)
        os.replace(tmp, out)
    return out


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv, ptxas_v="--ptxas" in sys.argv, tsan="--tsan" in sys.argv))
