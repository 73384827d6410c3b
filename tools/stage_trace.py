"""Per-stage clock64 timeline of the fused kernel (CTA 0, group 0, each warp):
wait -> (mbarrier satisfied) -> epilogue -> hand-off -> issue, cycles."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synth  # noqa: E402
import paper_conf_sc_cui0czlzsmylg21_b200 as ab  # noqa: E402

L = ab.lib()
L.abacus_internal_set_trace.argtypes = [C.c_void_p]
buf = torch.zeros(16 + 4 * 12 * 6, dtype=torch.int64, device="cuda")
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
b = buf.cpu().numpy()[16:].reshape(4, 12, 6).astype(np.int64)
t0 = b[:, :, 0][b[:, :, 0] > 0].min()
print("warp stage   start   wait  epilog handoff  issue  (cycles; * = issuer)")
for w in range(4):
    for s in range(12):
        r = b[w, s]
        if r[0] == 0:
            continue
        print("%d %5d %8d %6d %6d %6d %6d %s" % (w, s, r[0] - t0, r[1] - r[0], r[2] - r[1], r[3] - r[2], r[4] - r[3],
                                               "*" if r[5] else ""))
per = b[:, 4:, :]
print("median over stages 4..11: wait %.0f epilogue %.0f handoff %.0f issue %.0f; stage period %.0f" % (
    np.median(per[:, :, 1] - per[:, :, 0]), np.median(per[:, :, 2] - per[:, :, 1]),
    np.median(per[:, :, 3] - per[:, :, 2]), np.median(per[:, :, 4] - per[:, :, 3]),
    np.median(np.diff(per[:, :, 0], axis=1))))
ab.abacus_destroy(ctx)
