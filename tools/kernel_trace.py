"""In-kernel timeline of the fused tc kernel (CTA 0, %globaltimer, ns):
0 entry, 1 weights staged, 2 tables + TMEM ready, 3 tile loop done,
4 TMEM freed, 5 CTA result published, 6 last-CTA reduce done, 7 mapped publish done."""
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
stamps = torch.zeros(12, dtype=torch.int64, device="cuda")
ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
ab.abacus_load_predictor(ctx, synth.weights(1), ab.ABACUS_FP16)
g = ab.make_grid(synth.cfg4_grid())
H = synth.cfg4_headroom()
L.abacus_internal_set_trace(stamps.data_ptr())
names = ["staged", "tables+tmem", "tiles", "dealloc", "cta publish", "5->8 fence", "8->9 loads", "9->10 decode", "10->6 rest", "6->7 mapped"]
for count in [0, 1280, 128000, 1280000]:
    rows = []
    for i in range(30):
        stamps.zero_()
        torch.cuda.synchronize()
        ab.abacus_search_grid(ctx, g, H, 10**9, count)
        torch.cuda.synchronize()
        s = stamps.cpu().numpy().astype(np.int64)
        if i >= 5 and s[6] != 0:
            o = [s[1]-s[0], s[2]-s[1], s[3]-s[2], s[4]-s[3], s[5]-s[4], s[8]-s[5], s[9]-s[8], s[10]-s[9], s[6]-s[10], s[7]-s[6]]
            rows.append(o)
    if not rows:
        print("count %8d: CTA 0 never last" % count)
        continue
    m = np.median(np.array(rows), axis=0) / 1e3
    print("count %8d: " % count + "  ".join("%s %.2f" % (n, v) for n, v in zip(names, m)) + "  total %.2f us" % m.sum())
L.abacus_internal_set_trace(None)
ab.abacus_destroy(ctx)
