"""Build libdysel.so in-tree for sm_100a (nvcc 12.9), no torch involved.

    python -m paper_conf_asplos_changkh16_b200.build [--verbose]

Compiles csrc/*.cu with `-gencode arch=compute_100a,code=sm_100a -lineinfo
-O3` into objects under build/, links them with NCCL into
paper_conf_asplos_changkh16_b200/libdysel.so.  Rebuilds only what changed.
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INC = os.path.join(ROOT, "include")
OBJ = os.path.join(ROOT, "build", "obj")
LIB = os.path.join(HERE, "libdysel.so")
SOURCES = ["runtime.cu", "spmv.cu", "spmv_probe.cu", "spmv_prep.cu", "spmv_f2.cu", "sgemm.cu", "comm.cu", "iterate.cu", "stencil.cu", "spmtv.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
         "-I", INC, "-I", CSRC]


def _deps():
    hdrs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    hdrs += [os.path.join(INC, f) for f in os.listdir(INC)]
    return max(os.path.getmtime(h) for h in hdrs)


RDC = {"spmv.cu", "spmtv.cu"}   # the switch kernel's device-side launch (A-42) needs relocatable device code


def _compile(src, verbose, obj_dir=None, defines=()):
    obj = os.path.join(obj_dir or OBJ, src.replace(".cu", ".o"))
    path = os.path.join(CSRC, src)
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(path), _deps()):
        return obj, ""
    cmd = [NVCC, *ARCH, *FLAGS, *[f"-D{d}" for d in defines], *(["-rdc=true"] if src in RDC else []), "-c", path,
           "-o", obj]
    if verbose:
        cmd += ["-Xptxas", "-v"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    return obj, r.stderr


def build(verbose: bool = False, defines=(), out=None) -> str:
    """defines / out: an A/B build of the same sources with -D defines into
    another library path (objects under build/obj-<tag>); the product library
    is the default build."""
    lib = out or LIB
    obj_dir = OBJ if not defines else OBJ + "-" + "-".join(d.replace("=", "") for d in defines)
    os.makedirs(obj_dir, exist_ok=True)
    with cf.ThreadPoolExecutor(len(SOURCES)) as ex:
        results = list(ex.map(lambda s: _compile(s, verbose, obj_dir, defines), SOURCES))
    objs = [o for o, _ in results]
    if verbose:
        for _, log in results:
            if log:
                sys.stderr.write(log)
    if not os.path.exists(lib) or os.path.getmtime(lib) < max(os.path.getmtime(o) for o in objs):
        rdc = [o for o in objs if os.path.basename(o).replace(".o", ".cu") in RDC]
        dlink = os.path.join(obj_dir, "dlink.o")
        r = subprocess.run([NVCC, *ARCH, "-Xcompiler", "-fPIC", "-dlink", *rdc, "-o", dlink, "-lcudadevrt"],
                           capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"device link failed:\n{r.stderr}")
        cmd = [NVCC, *ARCH, "-shared", "-o", lib, *objs, dlink, "-lcudadevrt", "-ldl"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr}")
    return lib


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--verbose", action="store_true")
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-D", dest="defines", action="append", default=[], help="A/B build: extra -D define")
    ap.add_argument("--out", default=None, help="A/B build: library path")
    a = ap.parse_args()
    if a.force and os.path.isdir(OBJ):
        for f in os.listdir(OBJ):
            os.remove(os.path.join(OBJ, f))
    print(build(a.verbose, tuple(a.defines), a.out))
