"""Multi-process (world_size 2, gloo, CPU) coverage of the sharded sweep's host
logic: contiguous shards [floor(rT/G), floor((r+1)T/G)) partition the index
space, and one max collective over the per-rank best keys reproduces the
unsharded selection.  The per-rank search is the fp64 oracle
here (no GPU); the GPU path runs the same shard_range + combine."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, grid, H, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        params = synth.weights(1)
        T = oracle.grid_size(grid)
        first, count = ab.shard_range(T, rank, world)
        r, _, _, _ = oracle.sweep(params, grid, H, first=first, count=count)
        key = torch.tensor([r.best_key], dtype=torch.int64)
        dist.all_reduce(key, op=dist.ReduceOp.MAX)
        ev = torch.tensor([r.evaluated], dtype=torch.int64)
        dist.all_reduce(ev, op=dist.ReduceOp.SUM)
        # the NCCL bootstrap pattern of nccl_comm_from_process_group: rank 0's
        # 128 id bytes reach every rank intact
        blob = [bytes(range(128)) if rank == 0 else bytes(128)]
        dist.broadcast_object_list(blob, src=0)
        q.put((rank, int(key.item()), int(ev.item()), blob[0] == bytes(range(128)), first, count))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_sharded_sweep_combine_gloo(world):
    grid = [synth.GridSlot(1, 1, 8, 0, 1, 60, 1), synth.GridSlot(5, 1, 8, 0, 1, 40, 1),
            synth.GridSlot(7, 100, 4, 64, 100, 140, 1)]
    params = synth.weights(1)
    _, y, _, _ = oracle.sweep(params, grid, 0.0, want_y=True)
    import numpy as np
    H = float(np.float32(np.median(y)))
    full, _, _, _ = oracle.sweep(params, grid, H)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, grid, H, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    T = oracle.grid_size(grid)
    res.sort()
    assert res[0][4] == 0 and sum(r[5] for r in res) == T
    for i in range(world - 1):
        assert res[i][4] + res[i][5] == res[i + 1][4]       # contiguous shards
    for rank, key, ev, ok, _, _ in res:
        assert key == full.best_key and ev == T and ok


def test_shard_range_partitions():
    for T in (1, 7, 5043, 9_188_218_208):
        for G in (1, 2, 3, 4, 8):
            parts = [ab.shard_range(T, r, G) for r in range(G)]
            assert parts[0][0] == 0 and sum(c for _, c in parts) == T
            assert all(parts[i][0] + parts[i][1] == parts[i + 1][0] for i in range(G - 1))
            assert max(c for _, c in parts) - min(c for _, c in parts) <= 1
