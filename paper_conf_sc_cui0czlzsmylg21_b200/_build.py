"""Build the CUDA library in-tree with nvcc for sm_100a (no JIT cache)."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libabacus.so")
PROBE_LIB = os.path.join(HERE, "libabacus_probe.so")
SOURCES = ["abacus.cu", "kernels_simt.cu", "kernels_tc.cu", "kernels_train.cu"]
HEADERS = ["common.cuh", "device_common.cuh", "internal.h", "tc_ptx.cuh"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared"]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS]
    deps.append(os.path.join(os.path.dirname(HERE), "include", "abacus.h"))
    if force or _stale(LIB, deps):
        # one nvcc per translation unit, in parallel (no device code crosses files:
        # the kernels' helpers are header-inline), then one link
        import tempfile
        with tempfile.TemporaryDirectory() as tmp:
            objs, procs = [], []
            cflags = [f for f in FLAGS if f != "-shared"]
            for f in SOURCES:
                o = os.path.join(tmp, f + ".o")
                cmd = [NVCC] + ARCH + cflags + ["-c", "-o", o, os.path.join(CSRC, f)]
                if verbose:
                    print(" ".join(cmd))
                procs.append((subprocess.Popen(cmd), cmd))
                objs.append(o)
            for p, cmd in procs:
                if p.wait() != 0:
                    raise subprocess.CalledProcessError(p.returncode, cmd)
            cmd = [NVCC] + ARCH + ["-shared", "-Xcompiler", "-fPIC", "-o", LIB] + objs + ["-ldl"]
            if verbose:
                print(" ".join(cmd))
            subprocess.check_call(cmd)
    pdeps = [os.path.join(CSRC, "probe_umma.cu"), os.path.join(CSRC, "tc_ptx.cuh")]
    if force or _stale(PROBE_LIB, pdeps):
        cmd = [NVCC] + ARCH + FLAGS + ["-o", PROBE_LIB, os.path.join(CSRC, "probe_umma.cu")]
        subprocess.check_call(cmd)
    return LIB
