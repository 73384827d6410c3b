"""bench.py's N > 1 path on a one-GPU box: torchrun with two or three ranks, all on
cuda:0 (test mode ABACUS_BENCH_SHARE_GPU=1: gloo for the torch.distributed
plumbing, the sweep combined inside the search kernel over the two processes'
peer mailboxes, CUDA IPC).  Rank 0 alone prints one line; the config-4 sweep
split into 2 or 3 contiguous shards must select exactly what one unsharded
abacus_search_grid selects."""
import json
import os
import socket
import subprocess
import sys

import pytest

import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("nproc", [2, 3])
def test_bench_ranks_share_one_gpu_peer_combine(nproc):
    env = dict(os.environ, ABACUS_BENCH_SHARE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(nproc),
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", str(nproc),
           "--steps", "3", "--warmup", "3", "--combine", "peer", "--no-cpu-baseline", "--no-decisions"]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [l for l in p.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, p.stdout[:2000]
    d = json.loads(lines[0])
    assert d["n_gpus"] == nproc and d["config"]["shared_gpu_test_mode"] is True
    assert d["config"]["combine"] == "peer"
    T = d["config"]["candidates_per_step"]
    assert d["gpu_launches"] >= 3
    # the unsharded answer, one process
    ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
    try:
        ab.abacus_load_predictor(ctx, synth.weights(1), ab.ABACUS_FP16)
        ref = ab.abacus_search_grid(ctx, ab.make_grid(synth.cfg4_grid()), synth.cfg4_headroom(), 0, T)
    finally:
        ab.abacus_destroy(ctx)
    sel = d["selected"]
    assert (sel["key"], sel["index"], sel["end_op"]) == (ref.key, ref.index, list(ref.end_op))
    assert abs(sel["pred_ms"] - ref.pred_ms) == 0.0
