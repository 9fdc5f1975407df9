"""Build libsmiler.so (the C-ABI CUDA library) in-tree with nvcc for sm_100a.

    python -m paper_conf_sigmod_zhout15_b200.build [--force] [--verbose]

Each .cu is compiled to an object in parallel, then linked into
paper_conf_sigmod_zhout15_b200/libsmiler.so with the CUDA runtime linked
statically (so the library does not depend on which libcudart torch loads).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libsmiler.so")
BUILD = os.path.join(HERE, "_build")
ALU_BENCH = os.path.join(BUILD, "alu_bench")
SOURCES = ["smiler.cu", "dtw.cu", "predict.cu"]
HEADERS = ["internal.h", "kernels.cuh", "lb.cuh", os.path.join("..", "..", "include", "smiler.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "-Xcompiler", "-Werror=return-type",
         "--expt-relaxed-constexpr", "-I", os.path.join(ROOT, "include")]
# tuning experiments only (tools/): extra -D knobs, e.g. "-DSMILER_GS_MINB=3"
FLAGS += os.environ.get("SMILER_EXTRA_NVFLAGS", "").split()


def _stale(target: str, deps) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS]
    objs, jobs = [], []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(BUILD, src.replace(".cu", ".o"))
        objs.append(o)
        if force or _stale(o, [s, *hdrs, __file__]):
            cmd = [NVCC, *ARCH, *FLAGS, "-c", s, "-o", o]
            if verbose:
                cmd.insert(1, "-Xptxas=-v")
            jobs.append(cmd)

    def run(cmd):
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed:\n%s\n%s%s" % (" ".join(cmd), r.stdout, r.stderr))
        return r.stderr

    with cf.ThreadPoolExecutor(max_workers=len(SOURCES)) as ex:
        for err in ex.map(run, jobs):
            if verbose and err:
                sys.stderr.write(err)
    if force or jobs or _stale(LIB, objs):
        tmp = LIB + ".tmp%d" % os.getpid()
        run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs])
        os.replace(tmp, LIB)
    ab_src = os.path.join(CSRC, "alu_bench.cu")
    if force or _stale(ALU_BENCH, [ab_src]):
        run([NVCC, *ARCH, "-O3", "-lineinfo", "-o", ALU_BENCH, ab_src])
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv))
