"""Build libfastt.so in-tree with nvcc for sm_100a (no JIT, no torch extension).
Each translation unit compiles to an object in parallel (relocatable device
code is not needed: no kernel calls across files), then one link.  The two
simulation kernels' template instances are split by device-count width GSH:
k_sim_inst.cu is compiled once per GSH = 0..5, k_sim_lane_inst.cu once per
(GSH, memory mode MM = 0..2)."""
from __future__ import annotations

import os
import subprocess
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
_C = os.path.join(HERE, "csrc")
SRCS = [os.path.join(_C, f) for f in ("fastt_abi.cu", "k_prep.cu", "k_sim.cu", "k_sim_lane.cu", "k_fit.cu",
                                      "k_sim_inst.cu", "k_sim_lane_inst.cu", "k_lane_pk_inst.cu")]
# (source, extra flags): one object per unit
UNITS = ([(os.path.join(_C, "k_sim_lane_inst.cu"), ["-DFASTT_GSH=%d" % g, "-DFASTT_MM=%d" % m])
          for g in (5, 4, 3, 2, 1, 0) for m in range(3)] +
         [(os.path.join(_C, "k_sim_inst.cu"), ["-DFASTT_GSH=%d" % g]) for g in (5, 4, 3, 2, 1, 0)] +
         [(os.path.join(_C, "k_lane_pk_inst.cu"), ["-DFASTT_GSH=%d" % g]) for g in (5, 4, 3, 2, 1, 0)] +
         [(s, []) for s in SRCS[:5]])
DEPS = SRCS + [os.path.join(_C, f) for f in ("fastt_internal.cuh", "sim_common.cuh", "k_sim_body.cuh",
                                             "k_sim_lane_body.cuh", "k_lane_pk.cuh")] + [os.path.join(ROOT, "include", "fastt.h")]
OUT = os.path.join(HERE, "libfastt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CFLAGS = ARCH + ["-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-I" + os.path.join(ROOT, "include")]
# launch-shape overrides for tuning experiments (defaults live in fastt_internal.cuh)
CFLAGS += ["-D%s=%s" % (k, os.environ[k]) for k in ("SIM_MINB", "SIM_MINB_TOPO", "SIM_BLOCK", "LANE_MINB", "LANE_BLOCK") if os.environ.get(k)]
FLAGS = CFLAGS + ["-shared"]  # (single-command form, kept for tools)


OBJ_DIR = os.path.join(HERE, ".objs")  # per-unit objects kept between builds (git-ignored)
_ABI_DEPS = [os.path.join(_C, "fastt_abi.cu"), os.path.join(_C, "fastt_internal.cuh"),
             os.path.join(ROOT, "include", "fastt.h")]


_HDRS = [d for d in DEPS if not d.endswith(".cu")]


def _unit_deps(src):
    # fastt_abi.cu includes only the ABI header and fastt_internal.cuh; every
    # kernel unit is taken to depend on every header
    return _ABI_DEPS if os.path.basename(src) == "fastt_abi.cu" else [src] + _HDRS


def build(force: bool = False, verbose: bool = False, out: str = OUT) -> str:
    if not force and os.path.exists(out) and all(os.path.getmtime(out) >= os.path.getmtime(d) for d in DEPS):
        return out
    os.makedirs(OBJ_DIR, exist_ok=True)
    objs = [os.path.join(OBJ_DIR, "%02d_%s_%s.o" % (k, os.path.basename(u[0]), "_".join(u[1]) or "x"))
            for k, u in enumerate(UNITS)]
    stamp = os.path.join(OBJ_DIR, "flags")
    if not os.path.exists(stamp) or open(stamp).read() != " ".join(CFLAGS):
        force = True

    def cc(pair):
        (src, extra), obj = pair
        if not force and not verbose and os.path.exists(obj) and \
                all(os.path.getmtime(obj) >= os.path.getmtime(d) for d in _unit_deps(src)):
            return
        tmpo = obj + ".tmp%d" % os.getpid()
        cmd = [NVCC] + CFLAGS + extra + (["-Xptxas", "-v"] if verbose else []) + ["-c", src, "-o", tmpo]
        subprocess.check_call(cmd)
        os.replace(tmpo, obj)

    with ThreadPoolExecutor(max_workers=min(len(UNITS), os.cpu_count() or 4)) as ex:
        list(ex.map(cc, zip(UNITS, objs)))
    with open(stamp, "w") as f:
        f.write(" ".join(CFLAGS))
    tmp = out + ".tmp%d" % os.getpid()
    subprocess.check_call([NVCC] + ARCH + ["-shared", "-o", tmp] + objs)
    os.replace(tmp, out)
    return out


ALU_PEAK_SRC = os.path.join(ROOT, "tools", "alu_peak.cu")
ALU_PEAK = os.path.join(HERE, "alu_peak")


def build_alu_peak(force: bool = False) -> str:
    """the int32 pipe microbenchmark bench.py runs for its roofline peak"""
    if force or not os.path.exists(ALU_PEAK) or os.path.getmtime(ALU_PEAK) < os.path.getmtime(ALU_PEAK_SRC):
        tmp = ALU_PEAK + ".tmp%d" % os.getpid()
        subprocess.check_call([NVCC] + ARCH + ["-O3", "-o", tmp, ALU_PEAK_SRC])
        os.replace(tmp, ALU_PEAK)
    return ALU_PEAK


if __name__ == "__main__":
    import sys
    print(build(force="-f" in sys.argv, verbose="-v" in sys.argv))
