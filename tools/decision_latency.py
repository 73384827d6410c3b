"""Per-decision latency through the C ABI (tools/decision_latency.c; no Python
on the timed path).  Writes the input file, builds the driver, runs it.

  python tools/decision_latency.py --config cfg2|cfg3 --space grid|chain|auto [--precision fp16]
"""
import argparse
import json
import os
import struct
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_sc_cui0czlzsmylg21_b200 import _build  # noqa: E402

SPACE = {"grid": 0, "chain": 1, "auto": 2, "mway": 3}
PREC = {"fp32": 0, "bf16": 1, "fp16": 2}


def build_driver():
    src = os.path.join(ROOT, "tools", "decision_latency.c")
    exe = os.path.join(ROOT, "tools", "decision_latency")
    lib = _build.build()
    if not os.path.exists(exe) or os.path.getmtime(exe) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-I", os.path.join(ROOT, "include"), "-o", exe, src,
                               "-L", os.path.dirname(lib), "-labacus", "-Wl,-rpath," + os.path.dirname(lib)])
    return exe


def write_input(path, decs, precision, space, budget, warm):
    p = synth.weights(1)
    with open(path, "wb") as f:
        f.write(struct.pack("<i", synth.N_MODELS))
        f.write(struct.pack("<%di" % synth.N_MODELS, *[int(v) for v in synth.OPS_PER_MODEL]))
        f.write(struct.pack("<i", p.size))
        f.write(p.astype("<f4").tobytes())
        f.write(struct.pack("<iiQii", precision, space, budget, len(decs), warm))
        for qs, now, infl in decs:
            f.write(struct.pack("<idd", len(qs), now, infl))
            for q in qs:
                f.write(struct.pack("<iiiidd", q.model_id, q.next_op, q.batch, q.seqlen, q.qos_ms, q.t_start_ms))


def run(config="cfg2", space="grid", precision="fp16", n=10_000, warm=100, budget=4_194_304, batch=0):
    exe = build_driver()
    decs = synth.cfg2_decisions(n + warm) if config == "cfg2" else synth.cfg3_decisions(n + warm)
    path = "/tmp/abacus_dec_%s_%s.bin" % (config, space)
    write_input(path, decs, PREC[precision], SPACE[space], budget, warm)
    out = subprocess.check_output([exe, path] + ([str(batch)] if batch else [])).decode()
    d = json.loads(out)
    d.update({"config": config, "space": space, "precision": precision,
              "budget": budget if space == "auto" else None, "ways": budget if space == "mway" else None,
              "path": "C ABI (%s), host steady clock around each call" % (
                  "abacus_search_batch" if batch else "abacus_search")})
    return d


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="cfg2")
    ap.add_argument("--space", default="grid")
    ap.add_argument("--precision", default="fp16")
    ap.add_argument("-n", type=int, default=10_000)
    ap.add_argument("--budget", type=int, default=4_194_304, help="AUTO budget, or the ways of mway")
    ap.add_argument("--batch", type=int, default=0, help="decisions per abacus_search_batch call (0: single)")
    a = ap.parse_args()
    print(json.dumps(run(a.config, a.space, a.precision, a.n, budget=a.budget, batch=a.batch)))
