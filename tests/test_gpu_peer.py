"""GPU tests of the in-kernel cross-GPU combine (a6 over peer memory,
abacus_peer_comm_init): the last CTA of every rank's fused search writes its
record into every rank's mailbox and combines the records it finds in its own.

With one GPU, the ranks are ctxs on the same device: in one process (two
host threads, one ctx each; the mailboxes are plain device addresses) and in
two processes (the mailboxes are opened with CUDA IPC; the two processes'
kernels are time-sliced on the device, so the waiting last CTA must survive
being preempted).  Results must equal the unsharded search bit for bit and
the NCCL path's; a missing rank must fail after the timeout, not hang."""
import os
import socket
import threading

import numpy as np
import pytest

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab
from gpu_util import EPS, Ctx, accept_key, stream

pytestmark = pytest.mark.gpu


def _same(a, b):
    return (a.status, a.key, a.index, a.evaluated, list(a.end_op), a.total_ops, np.float32(a.pred_ms).tobytes(),
            np.float32(a.pred_critical_only_ms).tobytes()) == \
           (b.status, b.key, b.index, b.evaluated, list(b.end_op), b.total_ops, np.float32(b.pred_ms).tobytes(),
            np.float32(b.pred_critical_only_ms).tobytes())


def _comms(ctxs):
    blobs = [ab.abacus_peer_export(c.h) for c in ctxs]
    return [ab.abacus_peer_comm_init(c.h, len(ctxs), r, blobs) for r, c in enumerate(ctxs)]


def _parallel(fns):
    out = [None] * len(fns)
    err = []

    def run(i):
        try:
            out[i] = fns[i]()
        except Exception as e:  # noqa: BLE001
            err.append(e)
    ths = [threading.Thread(target=run, args=(i,)) for i in range(len(fns))]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=120)
    if err:
        raise err[0]
    return out


@pytest.mark.parametrize("prec", [ab.ABACUS_FP32, ab.ABACUS_FP16, ab.ABACUS_BF16], ids=["fp32", "fp16", "bf16"])
@pytest.mark.parametrize("G", [1, 2, 3])
def test_peer_combine_in_process(prec, G):
    """G ctxs on one device, one host thread each: every rank searches its shard
    with the peer combine; every rank returns the unsharded decision."""
    params = synth.weights(1)
    import torch
    ctxs = [Ctx(params=params, precision=prec) for _ in range(G)]
    streams = [torch.cuda.Stream() for _ in range(G)]  # every rank on its own stream: concurrent kernels
    for c, st in zip(ctxs, streams):
        ab.abacus_set_stream(c.h, st)
    comms = _comms(ctxs)
    try:
        # small grids: the G kernels (<= 148 / G CTAs each) are resident together
        g1 = [synth.GridSlot(1, 60, 8, 0, 60, 122, 1), synth.GridSlot(5, 1, 8, 0, 1, 40, 1)]
        g2 = [synth.GridSlot(2, 200, 8, 0, 200, 241, 1), synth.GridSlot(7, 220, 4, 64, 220, 243, 1),
              synth.GridSlot(5, 30, 4, 0, 30, 40, 1)]
        for slots in (g1, g2):
            T = oracle.grid_size(slots)
            grid = ab.make_grid(slots)
            _, y, _, _ = oracle.sweep(params, slots, 0.0, want_y=True)
            for q in (0.3, 0.8):
                H = float(np.float32(np.quantile(y, q)))
                whole = ab.abacus_search_grid(ctxs[0].h, grid, H, 0, T)
                got = _parallel([lambda r=r: ab.abacus_search_grid(ctxs[r].h, grid, H, *ab.shard_range(T, r, G),
                                                                   comms[r]) for r in range(G)])
                for d in got:
                    assert _same(d, whole), (G, q)
        # scheduling decisions sharded over the ranks (abacus_search_sharded)
        for qs, now, infl in synth.cfg2_decisions(6):
            ref = ab.abacus_search(ctxs[0].h, qs, now, infl, ab.ABACUS_SPACE_GRID)
            got = _parallel([lambda r=r: ab.abacus_search_sharded(ctxs[r].h, qs, now, infl, ab.ABACUS_SPACE_GRID,
                                                                  2**40, comms[r]) for r in range(G)])
            for d in got:
                assert _same(d, ref)
            od = oracle.search(params, qs, now, infl, space=0, eps=EPS[prec])
            if od.status == 0 and ref.status == 0:
                assert accept_key(ref.key, od.maxkey_strict, od.maxkey_loose)
    finally:
        for cm in comms:
            ab.abacus_peer_comm_destroy(cm)
        for c in ctxs:
            c.close()
        del streams


def test_peer_combine_missing_rank_times_out():
    """Rank 1 never launches: rank 0's kernel gives up after the timeout and
    the call fails with E_NCCL instead of hanging; the ctx stays usable."""
    os.environ["ABACUS_PEER_TIMEOUT_MS"] = "300"
    try:
        params = synth.weights(1)
        ctxs = [Ctx(params=params, precision=ab.ABACUS_FP16) for _ in range(2)]
        comms = _comms(ctxs)
        slots = synth.cfg1_grids()[0][1]
        T = oracle.grid_size(slots)
        with pytest.raises(ab.AbacusError) as e:
            ab.abacus_search_grid(ctxs[0].h, ab.make_grid(slots), 10.0, 0, T // 2, comms[0])
        assert e.value.code == ab.ABACUS_E_NCCL
        d = ab.abacus_search_grid(ctxs[0].h, ab.make_grid(slots), 10.0, 0, T)
        assert d.evaluated == T
    finally:
        os.environ.pop("ABACUS_PEER_TIMEOUT_MS", None)
        for cm in comms:
            ab.abacus_peer_comm_destroy(cm)
        for c in ctxs:
            c.close()


def _ipc_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        params = synth.weights(1)
        ctx = ab.abacus_create(0, list(synth.OPS_PER_MODEL))
        ab.abacus_load_predictor(ctx, params, ab.ABACUS_FP16)
        comm = ab.peer_comm_from_process_group(ctx)   # CUDA IPC between the two processes
        slots = synth.cfg1_grids()[2][1]
        T = oracle.grid_size(slots)
        out = []
        for H in (8.0, 12.0, 20.0):
            d = ab.abacus_search_grid(ctx, ab.make_grid(slots), H, *ab.shard_range(T, rank, world), comm)
            w = ab.abacus_search_grid(ctx, ab.make_grid(slots), H, 0, T)
            out.append((bytes(d), bytes(w)))
        ab.abacus_peer_comm_destroy(comm)
        ab.abacus_destroy(ctx)
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_peer_combine_two_processes_ipc():
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in range(2):
        for d, w in res[r]:
            dd, ww = ab.abacus_decision_t.from_buffer_copy(d), ab.abacus_decision_t.from_buffer_copy(w)
            assert _same(dd, ww)
    assert [d for d, _ in res[0]] == [d for d, _ in res[1]]


def test_peer_combine_many_consecutive_launches():
    """200 back-to-back sharded decisions on 2 ranks (the mailbox banks alternate
    by launch parity; a rank may start launch k + 1 while the other still reads
    launch k's records)."""
    import torch
    params = synth.weights(1)
    ctxs = [Ctx(params=params, precision=ab.ABACUS_FP16) for _ in range(2)]
    streams = [torch.cuda.Stream() for _ in range(2)]
    for c, st in zip(ctxs, streams):
        ab.abacus_set_stream(c.h, st)
    comms = _comms(ctxs)
    try:
        decs = synth.cfg2_decisions(200)
        refs = [ab.abacus_search(ctxs[0].h, qs, now, infl, ab.ABACUS_SPACE_GRID) for qs, now, infl in decs]

        def rank_loop(r):
            return [ab.abacus_search_sharded(ctxs[r].h, qs, now, infl, ab.ABACUS_SPACE_GRID, 2**40, comms[r])
                    for qs, now, infl in decs]
        got = _parallel([lambda r=r: rank_loop(r) for r in range(2)])
        for r in range(2):
            for d, ref in zip(got[r], refs):
                assert _same(d, ref)
    finally:
        for cm in comms:
            ab.abacus_peer_comm_destroy(cm)
        for c in ctxs:
            c.close()
        del streams
