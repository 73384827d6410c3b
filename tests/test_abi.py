"""CPU checks of the C-ABI boundary: the library builds for sm_100a, loads,
exports every function include/abacus.h declares, and the Python binding's
struct layouts equal the C header's (compiled with gcc).  No compute calls."""
import ctypes as C
import os
import re
import subprocess
import tempfile

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "abacus.h")


@pytest.fixture(scope="module")
def built():
    from paper_conf_sc_cui0czlzsmylg21_b200 import _build
    _build.build()
    return _build.LIB


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(abacus_\w+)\s*\(", src)))


def test_header_declares_the_four_north_star_calls():
    f = declared_functions()
    for name in ("abacus_encode_candidates", "abacus_predict_batch", "abacus_select_group", "abacus_search"):
        assert name in f


def test_library_exports_every_declared_symbol(built):
    out = subprocess.check_output(["nm", "-D", "--defined-only", built]).decode()
    exported = set(re.findall(r"\bT (abacus_\w+)", out))
    missing = [f for f in declared_functions() if f not in exported]
    assert not missing, missing
    import paper_conf_sc_cui0czlzsmylg21_b200 as ab
    assert sorted(ab.EXPORTED) == declared_functions()
    lib = C.CDLL(built)
    for f in declared_functions():
        getattr(lib, f)


def test_library_is_sm100a_native(built):
    out = subprocess.check_output(["cuobjdump", "--list-elf", built]).decode()
    assert "sm_100a" in out
    sass = subprocess.check_output(["cuobjdump", "-sass", built]).decode()
    assert "UTCHMMA" in sass and "LDTM" in sass and "STTM" in sass   # tcgen05.mma / ld / st


def test_struct_layouts_match_header(built):
    import paper_conf_sc_cui0czlzsmylg21_b200 as ab
    prog = r'''
#include <stdio.h>
#include <stddef.h>
#include "abacus.h"
int main(void) {
  printf("%zu %zu %zu %zu %zu %zu %zu %zu %zu %zu\n", sizeof(abacus_slot_t), sizeof(abacus_grid_t),
         sizeof(abacus_group_t), sizeof(abacus_query_t), sizeof(abacus_decision_t),
         offsetof(abacus_decision_t, key), offsetof(abacus_decision_t, total_ops),
         offsetof(abacus_query_t, qos_ms), sizeof(abacus_variant_t), offsetof(abacus_variant_t, seqlen));
  return 0;
}'''
    with tempfile.TemporaryDirectory() as d:
        c = os.path.join(d, "s.c")
        open(c, "w").write(prog)
        exe = os.path.join(d, "s")
        subprocess.check_call(["gcc", "-I", os.path.dirname(HEADER), "-o", exe, c])
        got = [int(v) for v in subprocess.check_output([exe]).decode().split()]
    want = [C.sizeof(ab.abacus_slot_t), C.sizeof(ab.abacus_grid_t), C.sizeof(ab.abacus_group_t),
            C.sizeof(ab.abacus_query_t), C.sizeof(ab.abacus_decision_t), ab.abacus_decision_t.key.offset,
            ab.abacus_decision_t.total_ops.offset, ab.abacus_query_t.qos_ms.offset, C.sizeof(ab.abacus_variant_t),
            ab.abacus_variant_t.seqlen.offset]
    assert got == want


def test_calls_fail_loudly_without_gpu(built):
    """No CPU fallback: creating a context on a GPU-less host is an error."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_sc_cui0czlzsmylg21_b200 as ab
    with pytest.raises(ab.AbacusError):
        ab.abacus_create(0, [10, 20])
