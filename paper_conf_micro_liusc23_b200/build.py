"""Builds libphoton.so in-tree (sm_100a only) with nvcc.  Used by __graft_entry__.build() and the binding."""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
SO = os.path.join(HERE, "libphoton.so")
OBJ = os.path.join(HERE, "_obj")
# debug variant: the same sources with PHOTON_DEBUG=1 (device-side bounds checks that trap; tests/test_debug_build.py)
SO_DEBUG = os.path.join(HERE, "libphoton_debug.so")
OBJ_DEBUG = os.path.join(HERE, "_obj_debug")
SOURCES = ["abi.cu", "k_bbv3.cu", "k_types.cu", "k_match.cu", "k_stable.cu", "k_predict.cu", "k_pool.cu", "k_full.cu"]
HEADERS = ["common.cuh", "internal.h"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
         "-Xcompiler", "-fvisibility=hidden", "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include")]


def _mtime(p):
    return os.path.getmtime(p) if os.path.exists(p) else -1.0


def build(force: bool = False, verbose: bool = False, debug: bool = False) -> str:
    obj_dir, so_path = (OBJ_DEBUG, SO_DEBUG) if debug else (OBJ, SO)
    extra = ["-DPHOTON_DEBUG=1"] if debug else []
    os.makedirs(obj_dir, exist_ok=True)
    deps = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "photon.h")]
    dep_t = max(_mtime(d) for d in deps)
    jobs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(obj_dir, src.replace(".cu", ".o"))
        if force or _mtime(o) < max(_mtime(s), dep_t):
            jobs.append((s, o))

    def cc(job):
        s, o = job
        cmd = [NVCC, *FLAGS, *extra, "-c", s, "-o", o]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {s}:\n{r.stderr}")
        if verbose and r.stderr:
            sys.stderr.write(r.stderr)
        return o

    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        list(ex.map(cc, jobs))
    objs = [os.path.join(obj_dir, s.replace(".cu", ".o")) for s in SOURCES]
    if force or jobs or _mtime(so_path) < max(_mtime(o) for o in objs):
        tmp = so_path + ".tmp"
        cmd = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-Xcompiler", "-fPIC", *objs, "-o", tmp,
               "-lcudart_static", "-lrt", "-ldl", "-lpthread"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
        os.replace(tmp, so_path)
    return so_path


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True, debug="--debug" in sys.argv))
