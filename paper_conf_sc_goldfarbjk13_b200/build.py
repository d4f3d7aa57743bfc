"""Build libtt.so in-tree: nvcc for sm_100a (-gencode arch=compute_100a,code=sm_100a),
g++ for the host builders (-ffp-contract=off: pinned fp32 arithmetic, R0)."""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
INC = os.path.join(os.path.dirname(HERE), "include")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libtt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU = ["tt_api.cu", "kern_bh.cu", "kern_bh_group.cu", "kern_pc.cu", "kern_pc_split.cu", "kern_knn.cu", "kern_vp.cu", "kern_nn.cu", "kern_sort.cu", "kern_sched.cu", "kern_recursive.cu", "kern_stack.cu",
      "build_oct_gpu.cu", "build_kd_gpu.cu", "build_vp_gpu.cu", "build_nn_gpu.cu",
      "kern_integrate.cu", "kern_diag.cu"]
CPP = ["host_build.cpp", "pack.cpp"]
HDRS = ["tt_internal.h", "kern_common.cuh", "blob_cache.h", "build_common.cuh", "tt_check.cuh"]
# --checked: device-side bounds checks (tt_check.cuh) into libtt_checked.so
CHECKED = {"build": os.path.join(HERE, "_build_checked"), "lib": os.path.join(HERE, "libtt_checked.so"),
           "defs": ["-DTT_CHECKED"]}


def _newer(src_list, out):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in src_list)


def _compile(src: str, verbose: bool, build_dir: str = BUILD, defs=()) -> str:
    obj = os.path.join(build_dir, os.path.basename(src) + ".o")
    deps = [os.path.join(CSRC, src)] + [os.path.join(CSRC, h) for h in HDRS] + [os.path.join(INC, "tt.h")]
    if not _newer(deps, obj):
        return obj
    if src.endswith(".cu"):
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", INC,
               "--expt-relaxed-constexpr", "-c", os.path.join(CSRC, src), "-o", obj]
        if verbose:
            cmd += ["-Xptxas", "-v"]
        cmd += list(defs)
    else:
        cmd = ["g++", "-O3", "-std=c++17", "-fPIC", "-ffp-contract=off", "-fno-fast-math", "-Wall",
               "-I", INC, "-I", "/usr/local/cuda/include", "-c", os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    if verbose and r.stderr:
        sys.stderr.write(r.stderr)
    return obj


def build(verbose: bool = False, force: bool = False, checked: bool = False) -> str:
    build_dir = CHECKED["build"] if checked else BUILD
    lib = CHECKED["lib"] if checked else LIB
    defs = CHECKED["defs"] if checked else []
    os.makedirs(build_dir, exist_ok=True)
    if force:
        for f in os.listdir(build_dir):
            os.remove(os.path.join(build_dir, f))
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose, build_dir, defs), CU + CPP))
    if _newer(objs, lib):
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", lib + ".tmp", *objs]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
        os.replace(lib + ".tmp", lib)
    return lib


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv, force="-f" in sys.argv, checked="--checked" in sys.argv))
