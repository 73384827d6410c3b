"""GPU parity of the what-if sweep (batch size and
sequence length as swept grid dimensions) against the fp64
oracle's what-if (oracle.whatif, pinned in tests/test_oracle_pins.py).

* Per variant, the batched what-if launch must equal abacus_search_grid of the
  variant's own grid bit for bit (same per-row arithmetic), and be acceptable
  to the oracle (reading c18).
* The global best (max sum_n, then max index v T + t) must lie in the
  oracle's acceptance window lifted to global indices.
"""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import EPS, NAMES, Ctx, accept_key

pytestmark = pytest.mark.gpu
PRECS = [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16]


@pytest.fixture(scope="module")
def ctx():
    c = Ctx(params=synth.weights(1), precision=ab.ABACUS_FP32)
    yield c
    c.close()


def _cases():
    # config 1 (ResNet-50 + VGG-16) over the paper's batch sizes (Table 1: 1..32)
    g1 = synth.cfg1_grids()[0][1]
    v1 = [([b, b], [0, 0]) for b in (1, 2, 4, 8, 16, 32)]
    # 3 slots with a BERT: batch and sequence length of the BERT query swept
    g2 = [synth.GridSlot(2, 200, 8, 0, 200, 241, 1), synth.GridSlot(4, 180, 8, 0, 200, 220, 0),
          synth.GridSlot(7, 200, 4, 64, 200, 243, 1)]
    v2 = [([8, 8, b], [0, 0, s]) for b in (1, 4, 16) for s in (16, 128, 512)]
    # 4 slots, all absent allowed (16 presence patterns per variant)
    g3 = [synth.GridSlot(3, 330, 8, 0, 330, 360, 1), synth.GridSlot(4, 205, 8, 0, 205, 220, 1),
          synth.GridSlot(7, 220, 8, 128, 220, 243, 1), synth.GridSlot(8, 450, 4, 512, 450, 471, 1)]
    v3 = [([b, 8, 8, 4], [0, 0, 128, s]) for b in (2, 16) for s in (64, 512)]
    return [(g1, v1), (g2, v2), (g3, v3)]


@pytest.mark.parametrize("prec", PRECS, ids=[NAMES[p] for p in PRECS])
def test_whatif_matches_per_variant_grid_and_oracle(ctx, prec):
    ctx.load(ctx.params, prec)
    eps = EPS[prec]
    for ci, (slots, variants) in enumerate(_cases()):
        T = oracle.grid_size(slots)
        # headroom at the median of the first variant's predictions
        _, y, _, _ = oracle.sweep(ctx.params, slots, 0.0, want_y=True)
        for q in (0.1, 0.6):
            H = float(np.float32(np.quantile(y, q)))
            per, best, bv = ab.abacus_search_whatif(ctx.h, ab.make_grid(slots), variants, H)
            oper, (okey, ov, ot), (strict, loose) = oracle.whatif(ctx.params, slots, variants, H, eps=eps)
            for v, (bss, sls) in enumerate(variants):
                gv = [synth.GridSlot(s.model_id, s.start_op, bss[j], sls[j], s.end_lo, s.end_hi, s.allow_absent)
                      for j, s in enumerate(slots)]
                single = ab.abacus_search_grid(ctx.h, ab.make_grid(gv), H, 0, T)
                d = per[v]
                assert (d.status, d.key, list(d.end_op), d.total_ops, d.evaluated) == \
                       (single.status, single.key, list(single.end_op), single.total_ops, single.evaluated), (ci, v)
                if d.key:
                    assert np.float32(d.pred_ms) == np.float32(single.pred_ms)
                assert np.float32(d.pred_critical_only_ms) == np.float32(single.pred_critical_only_ms)
                assert accept_key(d.key, oper[v].maxkey_strict, oper[v].maxkey_loose), (ci, v, d.key)
            assert accept_key(best.key, strict, loose), (ci, q, best.key, strict, loose)
            assert best.evaluated == T * len(variants)
            if best.key:
                assert bv == best.index // T and per[bv].key & ((1 << 40) - 1) == best.index % T
                assert list(best.end_op) == list(per[bv].end_op)
                _, _, _, ope = oracle.sweep(ctx.params, [synth.GridSlot(s.model_id, s.start_op, variants[bv][0][j],
                                                                        variants[bv][1][j], s.end_lo, s.end_hi,
                                                                        s.allow_absent)
                                                         for j, s in enumerate(slots)],
                                            H, first=best.index % T, count=1, want_ope=True)
                assert list(best.end_op)[:len(slots)] == [int(o) for o in ope[0]]
            else:
                assert bv == -1 and strict == 0
    ctx.load(ctx.params, ab.ABACUS_FP32)


def test_whatif_errors(ctx):
    slots = synth.cfg1_grids()[0][1]
    g = ab.make_grid(slots)
    with pytest.raises(ab.AbacusError):
        ab.abacus_search_whatif(ctx.h, g, [], 10.0)
    with pytest.raises(ab.AbacusError):
        ab.abacus_search_whatif(ctx.h, g, [([0, 1], [0, 0])], 10.0)   # batch 0
    with pytest.raises(ab.AbacusError):
        ab.abacus_search_whatif(ctx.h, g, [([1, 1], [-1, 0])], 10.0)  # seqlen < 0
    big = synth.cfg4_grid()  # 9.19e9 candidates: 120 variants exceed 2^40 indices
    with pytest.raises(ab.AbacusError):
        ab.abacus_search_whatif(ctx.h, ab.make_grid(big), [([8, 8, 8, 4], [0, 0, 128, 512])] * 120, 30.0)


@pytest.mark.parametrize("prec", [ab.ABACUS_FP16, ab.ABACUS_BF16], ids=["fp16", "bf16"])
def test_whatif_large_grid_takes_per_variant_launches(ctx, prec):
    """Variant grids of >= 2^24 candidates run one fused search launch each:
    every variant equals abacus_search_grid of its grid, and the global best is
    the max over the variants' keys lifted to v T + t."""
    ctx.load(ctx.params, prec)
    slots = [synth.GridSlot(3, 200, 8, 0, 200, 360, 1), synth.GridSlot(4, 100, 8, 0, 100, 220, 1),
             synth.GridSlot(7, 100, 8, 128, 100, 243, 1), synth.GridSlot(8, 400, 4, 512, 400, 471, 1)]
    T = oracle.grid_size(slots)
    assert T >= 1 << 24
    variants = [([8, 8, 8, b], [0, 0, 128, 512]) for b in (1, 4, 16)]
    H = synth.cfg4_headroom()
    per, best, bv = ab.abacus_search_whatif(ctx.h, ab.make_grid(slots), variants, H)
    lifted = []
    for v, (bss, sls) in enumerate(variants):
        gv = [synth.GridSlot(s.model_id, s.start_op, bss[j], sls[j], s.end_lo, s.end_hi, s.allow_absent)
              for j, s in enumerate(slots)]
        single = ab.abacus_search_grid(ctx.h, ab.make_grid(gv), H, 0, T)
        assert (per[v].key, list(per[v].end_op), per[v].evaluated) == (single.key, list(single.end_op), T)
        k = per[v].key
        lifted.append(((k >> 40) << 40) | (v * T + (k & ((1 << 40) - 1))) if k else 0)
    assert best.key == max(lifted) and (bv == int(np.argmax(lifted)) if best.key else bv == -1)
    ctx.load(ctx.params, ab.ABACUS_FP32)


@pytest.mark.parametrize("prec", [ab.ABACUS_FP16, ab.ABACUS_BF16], ids=["fp16", "bf16"])
def test_whatif_small_radix_grids(ctx, prec):
    """Grids whose digits all have few options (2..23), so one tile advance
    (+128 rows) wraps several digits at once: the batch kernel's walker adds
    the advance as mixed-radix digits with one carry per digit, the single
    search divides by each radix.  Every variant must equal abacus_search_grid
    bit for bit and be acceptable to the oracle; the whole grid spans many
    tiles and a ragged tail."""
    ctx.load(ctx.params, prec)
    rng = np.random.default_rng(61)
    for it in range(12):
        k = int(rng.integers(2, 5))
        models = [int(m) for m in rng.choice(np.arange(1, 9), size=k, replace=False)]
        slots = []
        for m in models:
            L = synth.L(m)
            n = int(rng.integers(1, 23))
            lo = int(rng.integers(1, L - n + 2))
            slots.append(synth.GridSlot(m, lo, int(rng.choice([1, 8, 32])), synth.seqlen_for(m, 128), lo,
                                        lo + n - 1, int(rng.integers(0, 2))))
        T = oracle.grid_size(slots)
        _, y, _, _ = oracle.sweep(ctx.params, slots, 0.0, want_y=True)
        H = float(np.float32(np.quantile(y, rng.uniform(0.2, 0.9))))
        variants = [([int(b)] * k, [synth.seqlen_for(m, int(s)) for m in models])
                    for b, s in ((1, 16), (8, 128), (32, 512))]
        per, best, bv = ab.abacus_search_whatif(ctx.h, ab.make_grid(slots), variants, H)
        oper, _, (strict, loose) = oracle.whatif(ctx.params, slots, variants, H, eps=EPS[prec])
        for v, (bss, sls) in enumerate(variants):
            gv = [synth.GridSlot(s.model_id, s.start_op, bss[j], sls[j], s.end_lo, s.end_hi, s.allow_absent)
                  for j, s in enumerate(slots)]
            single = ab.abacus_search_grid(ctx.h, ab.make_grid(gv), H, 0, T)
            assert (per[v].key, list(per[v].end_op), per[v].evaluated) == \
                   (single.key, list(single.end_op), single.evaluated), (it, v, T)
            assert accept_key(per[v].key, oper[v].maxkey_strict, oper[v].maxkey_loose), (it, v)
        assert accept_key(best.key, strict, loose)
    ctx.load(ctx.params, ab.ABACUS_FP32)
