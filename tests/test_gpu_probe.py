"""Pin the tcgen05 operand layouts the tensor-core kernels assume (one MMA,
M=128 x N x K=16, A in TMEM, B in shared memory) against numpy on small
integers that are exact in fp16 and bf16.  Test-only probe library."""
import ctypes as C
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _lib():
    from paper_conf_sc_cui0czlzsmylg21_b200 import _build
    _build.build()
    L = C.CDLL(_build.PROBE_LIB)
    L.abacus_probe_mma.argtypes = [C.c_int, C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_void_p]
    return L


def _bits(v, fmt):
    v = np.asarray(v, dtype=np.float32)
    if fmt == 0:
        return v.astype(np.float16).view(np.uint16)
    return (v.view(np.uint32) >> 16).astype(np.uint16)  # exact small integers: truncation == RNE


@pytest.mark.parametrize("fmt", [0, 1])
@pytest.mark.parametrize("N", [32, 16])
def test_umma_layouts(fmt, N):
    L = _lib()
    rng = np.random.default_rng(fmt * 7 + N)
    A = rng.integers(-3, 4, size=(128, 16)).astype(np.float32)
    B = rng.integers(-2, 3, size=(N, 16)).astype(np.float32)
    ab = _bits(A, fmt).astype(np.uint32)
    words = np.ascontiguousarray((ab[:, 1::2] << 16) | ab[:, 0::2], dtype=np.uint32)   # k=2c low half
    bb = np.ascontiguousarray(_bits(B, fmt))
    want = A @ B.T
    res = {}
    for variant in range(4):
        out = np.zeros((128, N), dtype=np.float32)
        rc = L.abacus_probe_mma(fmt, variant, N, words.ctypes.data, bb.ctypes.data, out.ctypes.data)
        assert rc == 0
        res[variant] = out
    print({v: bool(np.array_equal(o, want * (2 if v == 3 else 1))) for v, o in res.items()})
    assert np.array_equal(res[0], want), "descriptor (LBO=128 K-dir, SBO=256 N-dir) / A packing"
    assert np.array_equal(res[2], want), "A at a TMEM column offset of 8"
    assert np.array_equal(res[3], 2 * want), "accumulate flag"


@pytest.mark.parametrize("fmt", [0, 1])
def test_umma_m128_n8(fmt):
    """M = 128 with N = 8 (the output layer's width): the MMA computes the 8
    columns and leaves the rest of the 32-column D region untouched."""
    L = _lib()
    rng = np.random.default_rng(5 + fmt)
    N = 8
    A = rng.integers(-3, 4, size=(128, 16)).astype(np.float32)
    B = rng.integers(-2, 3, size=(N, 16)).astype(np.float32)
    ab = _bits(A, fmt).astype(np.uint32)
    words = np.ascontiguousarray((ab[:, 1::2] << 16) | ab[:, 0::2], dtype=np.uint32)
    bb = np.ascontiguousarray(_bits(B, fmt))
    out = np.zeros((128, 32), dtype=np.float32)
    rc = L.abacus_probe_mma(fmt, 6, N, words.ctypes.data, bb.ctypes.data, out.ctypes.data)
    assert rc == 0
    assert np.array_equal(out[:, :8], A @ B.T)
    assert np.all(out[:, 8:] == -777.0)
