"""A short, seeded slice of tests/fuzz_parity.py in the GPU suite: random
grids, scheduling rounds (GRID / CHAIN / AUTO), batched rounds and what-if
sets in all three precisions against the fp64 oracle (reading c18), batches
bit-identical to the single calls.  The long run (10 minutes, 0 failures) is
recorded in profiles/r2_fuzz.txt."""
import pytest

import fuzz_parity

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("seed", [7, 8])
def test_random_parity_slice(seed):
    n, fails = fuzz_parity.run(seed, iterations=6)
    assert fails == 0, n
    assert n["grid"] > 0 and n["round"] == 48 and n["batch"] == 32 and n["whatif"] > 0
