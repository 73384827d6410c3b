"""Probe the TMEM layout of an f16 accumulator (tcgen05.mma kind::f16 with
c_format F16): which 32-bit columns / halves hold D[m, n]."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
from paper_conf_sc_cui0czlzsmylg21_b200 import _build  # noqa: E402

L = C.CDLL(_build.PROBE_LIB)
L.abacus_probe_mma.argtypes = [C.c_int, C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p]
rng = np.random.default_rng(3)
for N in (32, 16):
    A = rng.integers(-3, 4, size=(128, 16)).astype(np.float32)
    B = rng.integers(-2, 3, size=(N, 16)).astype(np.float32)
    ab = A.astype(np.float16).view(np.uint16).astype(np.uint32)
    words = np.ascontiguousarray((ab[:, 1::2] << 16) | ab[:, 0::2], dtype=np.uint32)
    bb = np.ascontiguousarray(B.astype(np.float16).view(np.uint16))
    want = A @ B.T
    for variant in (4, 5):
        out = np.zeros((128, N), dtype=np.float32)
        rc = L.abacus_probe_mma(0, variant, N, words.ctypes.data, bb.ctypes.data, out.ctypes.data)
        w = out.view(np.uint32)
        lo = (w & 0xFFFF).astype(np.uint16).view(np.float16).astype(np.float32)
        hi = (w >> 16).astype(np.uint16).view(np.float16).astype(np.float32)
        f = 2 if variant == 5 else 1
        print("N", N, "variant", variant, "rc", rc)
        print("  row0 words", [hex(x) for x in w[0, :min(N, 16)]])
        print("  want row0", (f * want[0]).tolist())
        packed = np.zeros((128, N), np.float32)
        packed[:, 0::2] = lo[:, :N // 2]
        packed[:, 1::2] = hi[:, :N // 2]
        print("  packed(col c = n 2c lo, 2c+1 hi):", bool(np.array_equal(packed, f * want)))
        print("  one-per-col low half:", bool(np.array_equal(lo, f * want)))
