"""Build libfastt.so in-tree with nvcc for sm_100a (no JIT, no torch extension)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
SRCS = [os.path.join(HERE, "csrc", f) for f in ("fastt_abi.cu", "k_prep.cu", "k_sim.cu", "k_fit.cu")]
DEPS = SRCS + [os.path.join(HERE, "csrc", "fastt_internal.cuh"), os.path.join(ROOT, "include", "fastt.h")]
OUT = os.path.join(HERE, "libfastt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC",
         "-shared", "-I" + os.path.join(ROOT, "include")]
# launch-shape overrides for tuning experiments (defaults live in fastt_internal.cuh)
FLAGS += ["-D%s=%s" % (k, os.environ[k]) for k in ("SIM_MINB", "SIM_BLOCK") if os.environ.get(k)]


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and os.path.exists(OUT) and all(os.path.getmtime(OUT) >= os.path.getmtime(d) for d in DEPS):
        return OUT
    tmp = OUT + ".tmp%d" % os.getpid()
    cmd = [NVCC] + FLAGS + (["-Xptxas", "-v"] if verbose else []) + ["-o", tmp] + SRCS
    subprocess.check_call(cmd)
    os.replace(tmp, OUT)
    return OUT


if __name__ == "__main__":
    import sys
    print(build(force="-f" in sys.argv, verbose="-v" in sys.argv))
