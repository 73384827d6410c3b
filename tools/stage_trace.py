"""Per-stage clock64 timeline of the fused fp16 kernel (experiment build with
-DEXP_STAGETRACE; CTA 0, group 0, lane 0 of each of its 4 warps, iterations
64..79).  Stage s = 0,1,2: wait for layer s+1 (L1, L2, L3) -> epilogue -> hand-off
-> issue of the next layer; s = 3: wait for the output layer -> fold + walk ->
hand-off -> layer-1 issue of the next tiles.  Prints cycles per stage:
  mma  = issue (by the stage's issuer) -> mbarrier satisfied (warp's view)
  epi  = mbarrier satisfied -> this warp's operand stored
  hand = last warp stored -> issuer past the barrier
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402
import ctypes as C  # noqa: E402

L = ab.lib()
L.abacus_internal_set_trace.argtypes = [C.c_void_p]
NIT = 16
buf = torch.zeros(16 + NIT * 4 * 4 * 3, dtype=torch.int64, device="cuda")
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
ab.abacus_set_stream(ctx, st)
ab.abacus_load_predictor(ctx, synth.weights(1), ab.ABACUS_FP16)
g = ab.make_grid(synth.cfg4_grid())
T = 9188218208
for _ in range(3):
    ab.abacus_search_grid(ctx, g, synth.cfg4_headroom(), 0, T // 64)
L.abacus_internal_set_trace(buf.data_ptr())
ab.abacus_search_grid(ctx, g, synth.cfg4_headroom(), 0, T // 64)
torch.cuda.synchronize()
L.abacus_internal_set_trace(None)
b = buf.cpu().numpy()[16:].reshape(NIT, 4, 4, 3).astype(np.int64)  # it, warp, stage, (wait, stored, issued)
names = ["L1->L2", "L2->L3", "L3->out", "out->L1"]
rows = []
for it in range(1, NIT):
    for s in range(4):
        issuer = (0 + s) & 3  # group 0: issuer of hand-off position p is warp p
        t_issue = b[it, issuer, s, 2]
        # previous issue that this stage waits for: stage s-1 of the same iteration (or stage 3 of the previous)
        prev_s, prev_it = (s - 1, it) if s > 0 else (3, it - 1)
        t_prev_issue = b[prev_it, (0 + prev_s) & 3, prev_s, 2]
        t_wait = b[it, :, s, 0]
        t_store = b[it, :, s, 1]
        rows.append((s, t_wait.min() - t_prev_issue, (t_store - t_wait).mean(), t_issue - t_store.max(),
                     t_wait.max() - t_wait.min()))
r = np.array(rows, dtype=np.float64)
it_cycles = (b[NIT - 1, 0, 0, 0] - b[1, 0, 0, 0]) / (NIT - 2)
print("iteration (2 tiles per group): %.0f cycles" % it_cycles)
print("%-8s %8s %8s %8s %10s" % ("stage", "mma", "epi", "hand", "wake-skew"))
for s in range(4):
    m = r[r[:, 0] == s].mean(axis=0)
    print("%-8s %8.0f %8.0f %8.0f %10.0f" % (names[s], m[1], m[2], m[3], m[4]))
