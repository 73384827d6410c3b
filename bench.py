"""bench.py -- headline benchmark of the Abacus candidate-search hot path on B200.

Step = one abacus_search_grid over config 4 of BASELINE.json: the offline
exhaustive overlap sweep of ResNet-152 (bs 8), Inception-v3 (bs 8), BERT-base
(bs 8, seq 128) and BERT-large (bs 4, seq 512), 361*221*244*472 =
9,188,218,208 candidates (enumerate -> Fig.-8 encode -> MLP -> headroom mask ->
max key), sharded contiguously over the ranks with one NCCL all-gather of the
per-rank best (a6).  Metric: predictor candidates/s (whole job).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--precision fp16|bf16|fp32]
  python bench.py --impl reference ...   # the fp64 CPU oracle on a bounded sample

Inputs are synthetic (seeded weights of the paper's MLP shape, synth/); the
candidate space is generated on the fly inside the kernel, so there is no
input tensor to keep out of L2 -- the timed kernel reads only its ~20 KB of
weights and writes 48 bytes (config "l2": "no per-candidate memory traffic").
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

FLOP_PER_CAND = 2 * (synth.D * 32 + 32 * 32 + 32 * 32 + 32)  # 5,696 algorithmic FLOP (D = 24)
METRIC = "predictor candidates/sec (config 4 exhaustive overlap sweep, abacus_search_grid)"
PREC = {"fp32": 0, "bf16": 1, "fp16": 2}
DTYPE = {"fp32": "f32", "bf16": "bf16 (layers 2, 3, output bf16 operands, W3 hi+lo; layer-1 digit operand f16), f32 accum", "fp16": "f16 (layers 1-3: f16 accum; output: f32 accum)"}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured (MEASURED_PEAKS.json)"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback (B200_PROFILING.md)"


class Clocks:
    """SM clock and throttle-reason sampler during the timed region
    (B200_PROFILING.md clocks line): NVML every 10 ms from a thread (the
    device found by its PCI bus id), else `nvidia-smi -lms 200`."""

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None
        self.stop = None

    def _nvml_handle(self):
        import pynvml
        import torch
        pynvml.nvmlInit()
        pr = torch.cuda.get_device_properties(self.index)
        bus = "%08x:%02x:%02x.0" % (pr.pci_domain_id, pr.pci_bus_id, pr.pci_device_id)
        return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus)

    def _nvml_loop(self, nv, h):
        names = [("hw_slowdown", nv.nvmlClocksEventReasonHwSlowdown),
                 ("hw_thermal_slowdown", nv.nvmlClocksEventReasonHwThermalSlowdown),
                 ("sw_thermal_slowdown", nv.nvmlClocksEventReasonSwThermalSlowdown),
                 ("sw_power_cap", nv.nvmlClocksEventReasonSwPowerCap)]
        mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        while not self.stop.is_set():
            sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
            rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
            self.rows.append([str(sm), str(mx)] + ["Active" if rs & bit else "Not Active" for _, bit in names])
            self.stop.wait(0.01)

    def __enter__(self):
        try:
            nv, h = self._nvml_handle()
            self.stop = threading.Event()
            self.t = threading.Thread(target=self._nvml_loop, args=(nv, h), daemon=True)
            self.t.start()
            return self
        except Exception:  # noqa: BLE001 -- fall back to nvidia-smi
            self.stop = None
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + q,
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([v.strip() for v in line.split(",")])

    def __exit__(self, *a):
        if self.stop is not None:
            self.stop.set()
            self.t.join(timeout=5)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 2 + i and "Active" in r[2 + i]
                          and "Not" not in r[2 + i]})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def cpu_oracle_rate(params, slots, H, budget_s=12.0, chunk=100_000):
    """The fp64 oracle as it stands, 1 thread, on a contiguous sample of the
    config-4 grid starting at T/2 (all four services mostly present)."""
    import oracle
    T = oracle.grid_size(slots)
    first = T // 2
    n = 0
    t0 = time.perf_counter()
    while time.perf_counter() - t0 < budget_s:
        oracle.sweep(params, slots, H, first=first + n, count=chunk)
        n += chunk
    dt = time.perf_counter() - t0
    return n / dt, n, dt


def cpu_oracle_other_configs(params):
    """The fp64 oracle (1 thread, as it stands) on the other BASELINE configs
    (SURVEY §8(d)): config 1 (all five 5,043-candidate grids), config 2 (100
    3-way GRID decisions, oracle.search: a1 + exhaustive GRID + drop test),
    config 5 (1e5 instance-based predictions, oracle.mlp64_batch).  Each
    bounded to a few seconds."""
    import oracle
    out = {}
    t0 = time.perf_counter()
    n = 0
    for _, g in synth.cfg1_grids():
        r, _, _, _ = oracle.sweep(params, g, 15.0)
        n += r.evaluated
    dt = time.perf_counter() - t0
    out["cfg1"] = {"candidates": n, "s": dt, "candidates_per_s": n / dt}
    decs = synth.cfg2_decisions(100)
    t0 = time.perf_counter()
    n = 0
    for qs, now, infl in decs:
        n += oracle.search(params, qs, now, infl, space=0).evaluated
    dt = time.perf_counter() - t0
    out["cfg2"] = {"decisions": len(decs), "candidates": n, "s": dt, "candidates_per_s": n / dt,
                   "decisions_per_s": len(decs) / dt, "space": "grid"}
    G = synth.instance_samples(100_000, seed=15)
    X = oracle.encode_groups(synth.N_MODELS, synth.K_MAX, [g.slots for g in G])
    t0 = time.perf_counter()
    oracle.mlp64_batch(params, X)
    dt = time.perf_counter() - t0
    out["cfg5"] = {"predictions": len(G), "s": dt, "predictions_per_s": len(G) / dt}
    out["cores"] = 1
    return out


def cpu_oracle_rate_all_cores(params, slots, H, budget_s=8.0, chunk=50_000):
    """The same oracle on every host core the process may use: one Python
    thread per core, each sweeping its own contiguous sub-range (ctypes
    releases the GIL inside the C oracle)."""
    import threading
    import oracle
    ncores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    T = oracle.grid_size(slots)
    counts = [0] * ncores
    t0 = time.perf_counter()

    span = (T - T // 2) // ncores

    def work(w):
        first = T // 2 + w * span
        while time.perf_counter() - t0 < budget_s:
            r, _, _, _ = oracle.sweep(params, slots, H, first=first + counts[w], count=chunk)
            counts[w] += r.evaluated

    ths = [threading.Thread(target=work, args=(w,)) for w in range(ncores)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    dt = time.perf_counter() - t0
    n = sum(counts)
    return n / dt, n, dt, ncores


def arm_config(T, H, precision, world, combine="nccl"):
    """The workload both arms report (the reference arm times a bounded sample of it)."""
    how = ("NCCL all-gather of the per-rank results + finalize kernel" if combine == "nccl" else
           "combine inside the search kernel over peer mailboxes")
    return {"workload": "cfg4: 4-way exhaustive overlap sweep (ResNet-152, Inception-v3, BERT-base "
                        "seq128, BERT-large seq512), %d candidates" % T,
            "candidates_per_step": T, "headroom_ms": H, "precision": precision,
            "parallelism": "candidate shards x%d" % world + (", " + how if world > 1 else ""),
            "combine": combine if world > 1 else None,
            "l2": "no per-candidate memory traffic (candidates generated on chip)"}


def run_reference(args, rank, world):
    """The reference arm: the fp64 oracle as it stands, on every host core the
    process may use (one thread per core over its own contiguous sub-range of
    config 4; ctypes releases the GIL inside the C oracle).  A step is a
    bounded sample of the workload: per_thread candidates on each core."""
    if rank != 0:
        return
    import threading
    import oracle
    params = synth.weights(1)
    slots = synth.cfg4_grid()
    H = synth.cfg4_headroom()
    T = oracle.grid_size(slots)
    ncores = len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else (os.cpu_count() or 1)
    per_thread = 100_000
    # thread w sweeps its own contiguous range inside [T/2, T): starts spaced
    # (T - T/2) / ncores apart (always inside the grid, whatever the core
    # count); only the candidates the oracle actually evaluated are counted
    span = (T - T // 2) // ncores

    def step(i, counted):
        def work(w):
            first = T // 2 + w * span + (i * per_thread) % max(1, span - per_thread)
            r, _, _, _ = oracle.sweep(params, slots, H, first=first, count=per_thread)
            counted[w] = r.evaluated
        ths = [threading.Thread(target=work, args=(w,)) for w in range(ncores)]
        for th in ths:
            th.start()
        for th in ths:
            th.join()

    for i in range(args.warmup):
        step(i, [0] * ncores)
    counts = []
    t0 = time.perf_counter()
    for i in range(args.steps):
        c = [0] * ncores
        step(args.warmup + i, c)
        counts.append(sum(c))
    dt = time.perf_counter() - t0
    per_step = int(np.mean(counts))
    rate = sum(counts) / dt
    sample = "%d config-4 candidates per step: %d threads x %d contiguous, spread over [T/2, T)" % (
        per_step, ncores, per_thread)
    line = {"impl": "reference", "metric": METRIC, "value": rate, "unit": "candidates/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": dict(arm_config(T, H, "fp64 oracle", 1), reference_sample=sample),
            "cpu_baseline": {"value": rate, "unit": "candidates/s", "cores": ncores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": rate, "unit": "candidates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)


_JSON_OUT = None


def emit(line):
    """The one contract line goes to the process's original stdout; everything
    else printed at C level (NCCL's version banner, driver messages) was moved
    to stderr by main()."""
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    print(json.dumps(line), file=out, flush=True)


def main():
    global _JSON_OUT
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--precision", default="fp16", choices=list(PREC))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-decisions", action="store_true")
    ap.add_argument("--no-secondary", action="store_true", help="skip the bf16 / fp32 sweep keys")
    ap.add_argument("--combine", default="nccl", choices=["nccl", "peer"],
                    help="N > 1 sweep combine: NCCL all-gather + finalize kernel, or inside the search kernel")
    args = ap.parse_args()
    sys.stdout.flush()
    _JSON_OUT = os.fdopen(os.dup(1), "w")
    os.dup2(2, 1)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_sc_cui0czlzsmylg21_b200 as ab

    # test mode (tests/test_gpu_bench_multirank.py): every rank on cuda:0, gloo for the
    # torch.distributed plumbing, so the N > 1 path (shards, in-kernel peer combine,
    # max-over-ranks timing, one line from rank 0) runs on a one-GPU box.  NCCL refuses
    # two ranks on one GPU, so the NCCL legs are skipped there.  Never a bench number.
    share = os.environ.get("ABACUS_BENCH_SHARE_GPU") == "1" and world > 1
    if share:
        if args.combine != "peer":
            raise SystemExit("ABACUS_BENCH_SHARE_GPU=1 needs --combine peer (NCCL refuses two ranks on one GPU)")
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    params = synth.weights(1)
    slots = synth.cfg4_grid()
    H = synth.cfg4_headroom()
    grid = ab.make_grid(slots)
    T = 1
    for s in slots:
        T *= s.allow_absent + s.end_hi - s.end_lo + 1
    first, count = ab.shard_range(T, rank, world)

    ctx = ab.abacus_create(local, list(synth.OPS_PER_MODEL))
    ab.abacus_load_predictor(ctx, params, PREC[args.precision])
    # an explicit (non-legacy) stream shared by the library and the timing events
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    ab.abacus_set_stream(ctx, stream)
    ab.abacus_set_timing(ctx, True)
    comm = None
    if world > 1:
        comm = ab.nccl_comm_from_process_group(ctx) if args.combine == "nccl" else ab.peer_comm_from_process_group(ctx)

    for _ in range(args.warmup):
        d = ab.abacus_search_grid(ctx, grid, H, first, count, comm)
    # ---- device-timed region ------------------------------------------------
    launches0 = ab.abacus_kernel_launches(ctx)
    kernel_ms = []
    with Clocks(local) as clk:
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            d = ab.abacus_search_grid(ctx, grid, H, first, count, comm)
            kernel_ms.append(ab.abacus_last_kernel_ms(ctx))
        e1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    launches = ab.abacus_kernel_launches(ctx) - launches0
    elapsed = e0.elapsed_time(e1) / 1e3
    t = torch.tensor([elapsed, float(np.mean(kernel_ms))], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    elapsed, kms = float(t[0]), float(t[1])

    # ---- end to end through the public API (host structs in, host decision out) ----
    e2e_steps = max(2, args.steps // 2)
    if world > 1:
        dist.barrier()
    w0 = time.perf_counter()
    for _ in range(e2e_steps):
        d = ab.abacus_search_grid(ctx, grid, H, first, count, comm)
    w1 = time.perf_counter()
    te = torch.tensor([w1 - w0], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_rate = T * e2e_steps / float(te[0])

    # ---- per-decision sharded search (config 3 pure GRID, all ranks) --------
    sharded = None
    sharded_peer = None
    if not args.no_decisions:
        # at N = 1 through a one-rank NCCL communicator: the sharded path as it runs at N > 1
        if share:
            sharded = {"skipped": "ranks share one GPU (test mode): NCCL refuses that"}
        else:
            if world > 1:
                ncomm = comm if args.combine == "nccl" else ab.nccl_comm_from_process_group(ctx)
            else:
                ncomm = ab.abacus_nccl_comm_init(ctx, 1, 0, ab.abacus_nccl_unique_id())
            sharded = sharded_decision_latency(ab, ctx, ncomm, world, rank)
            if ncomm is not comm:
                ab.abacus_nccl_comm_destroy(ncomm)
        # the same decisions with the combine inside the search kernel (peer mailboxes,
        # CUDA IPC between the ranks' processes; at N = 1 a one-rank communicator).
        # Optional leg: every rank must agree that the communicator works (one probe
        # decision) before the loop, or all of them skip it.
        pcomm, err = None, None
        try:
            pcomm = ab.peer_comm_from_process_group(ctx) if world > 1 else \
                ab.abacus_peer_comm_init(ctx, 1, 0, [ab.abacus_peer_export(ctx)])
            qs, now, infl = synth.cfg3_decisions(1)[0]
            ab.abacus_search_sharded(ctx, qs, now, infl, ab.ABACUS_SPACE_GRID, 2**40, pcomm)
        except Exception as e:  # noqa: BLE001 -- report, do not fail the bench line
            err = repr(e)
        ok = err is None
        if world > 1:
            flag = torch.tensor([1 if ok else 0], dtype=torch.int32, device="cuda")
            dist.all_reduce(flag, op=dist.ReduceOp.MIN)
            ok = bool(flag.item())
        if ok:
            sharded_peer = sharded_decision_latency(ab, ctx, pcomm, world, rank, label="peer")
        else:
            sharded_peer = {"error": err or "the peer communicator failed on another rank"}
        if pcomm:
            ab.abacus_peer_comm_destroy(pcomm)

    # ---- per-decision latency (config 2, 3-way; 1 GPU each) -----------------
    dec = None
    if rank == 0 and not args.no_decisions:
        dec = decision_latency(ab, ctx, precision=args.precision)

    # ---- the other arithmetic paths on the same sweep (secondary keys) ------
    secondary = None
    whatif = None
    if world == 1 and not args.no_secondary:
        try:
            whatif = whatif_sweep(ab, ctx, slots, H, T)
        except Exception as e:  # noqa: BLE001 -- report, do not fail the bench line
            whatif = {"error": repr(e)}
        try:
            secondary = secondary_paths(ab, ctx, params, grid, H, T, args.precision, stream)
        except Exception as e:  # noqa: BLE001
            secondary = {"error": repr(e)}
            ab.abacus_load_predictor(ctx, params, PREC[args.precision])

    if rank == 0:
        pk, src = peaks()
        # the step is one kernel launch timed alone (clocks stay at max, no power cap in our
        # runs): the burst peak is the denominator; the sustained one is reported beside it.
        # fp16 dense = bf16 dense on B200 (B200_PROFILING.md nominal ratio 1).
        peak = pk["bf16_tflops"]
        achieved = FLOP_PER_CAND * count / (kms / 1e3) / 1e12
        traffic = None
        tp = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tp):
            with open(tp) as f:
                traffic = json.load(f).get("fused_" + args.precision)
        cpu = None
        cpu_all = None
        if not args.no_cpu_baseline:
            rate, n, dt = cpu_oracle_rate(params, slots, H)
            cpu = {"value": rate, "unit": "candidates/s", "cores": 1, "kind": "oracle",
                   "sample": "%d contiguous config-4 candidates from index T/2 (%.1f s, 1 thread)" % (n, dt)}
            ra, na, dta, nc = cpu_oracle_rate_all_cores(params, slots, H)
            cpu_all = {"value": ra, "unit": "candidates/s", "cores": nc, "kind": "oracle",
                       "sample": "%d config-4 candidates in %d contiguous ranges from T/2 (%.1f s, %d threads)"
                                 % (na, nc, dta, nc)}
            if world == 1:
                cpu["other_configs"] = cpu_oracle_other_configs(params)
        value = T * args.steps / elapsed
        line = {
            "metric": METRIC, "value": value, "unit": "candidates/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": elapsed / args.steps * 1e3, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": DTYPE[args.precision], "data": "synthetic",
            "config": dict(arm_config(T, H, args.precision, world, args.combine), shared_gpu_test_mode=share),
            "per_gpu": value / world,
            "selected": {"key": d.key, "index": d.index, "total_ops": d.total_ops, "pred_ms": d.pred_ms,
                         "end_op": list(d.end_op)},
            "roofline": {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel": "fused_tc_kernel" if args.precision != "fp32" else "fused_fp32_kernel",
                         "kernel_ms": kms, "flop_per_candidate": FLOP_PER_CAND, "peak_source": src + ", burst",
                         "frac_of_sustained": achieved / pk["bf16_tflops_sustained"]},
            "cpu_baseline": cpu,
            "cpu_baseline_all_cores": cpu_all,
            "e2e": {"value": e2e_rate, "unit": "candidates/s", "h2d_bytes_per_step": 120,
                    "d2h_bytes_per_step": 48},
            "gpu_launches": launches,
            "clocks": clk.summary(),
            "decision_latency": dec,
            "decision_latency_sharded": sharded,
            "decision_latency_sharded_peer": sharded_peer,
            "secondary_paths": secondary,
            "whatif": whatif,
        }
        emit(line)
    if world > 1:
        # rank 0 ran the single-GPU latency and CPU legs alone: every rank tears
        # down the library's communicator together (ncclCommDestroy finalizes)
        dist.barrier()
    if comm:
        (ab.abacus_nccl_comm_destroy if args.combine == "nccl" else ab.abacus_peer_comm_destroy)(comm)
    ab.abacus_destroy(ctx)
    if world > 1:
        dist.destroy_process_group()


def fp32_fma_peak_tflops(sm_mhz):
    """SIMT fp32 ceiling: 148 SMs x 128 FP32 lanes x 2 FLOP per FFMA x clock
    (B200_PROFILING.md unit counts)."""
    return 148 * 128 * 2 * sm_mhz * 1e6 / 1e12


def secondary_paths(ab, ctx, params, grid, H, T, headline, stream, steps=(("bf16", 6), ("fp32", 3))):
    """The same config-4 sweep in the other arithmetic paths (DESIGN.md r2):
    device time per sweep (CUDA events on the launching stream) and each
    path's own roofline: the tensor paths against the measured bf16 peak
    (fp16 = bf16 dense rate), fp32 SIMT against the FP32 FMA ceiling."""
    import torch
    out = {}
    pk, src = peaks()
    for name, n in steps:
        if name == headline:
            continue
        ab.abacus_load_predictor(ctx, params, PREC[name])
        d = ab.abacus_search_grid(ctx, grid, H, 0, T)  # warm-up
        kms = []
        with Clocks(0) as clk:
            for _ in range(n):
                d = ab.abacus_search_grid(ctx, grid, H, 0, T)
                kms.append(ab.abacus_last_kernel_ms(ctx))
        cs = clk.summary()
        k = float(np.mean(kms))
        achieved = FLOP_PER_CAND * T / (k / 1e3) / 1e12
        if name == "fp32":
            mhz = cs.get("sm_mhz") or 1965.0
            peak, unit, bound, psrc = fp32_fma_peak_tflops(mhz), "TFLOP/s", "alu", \
                "148 SM x 128 FFMA x 2 x %.0f MHz (median SM clock under load)" % mhz
        else:
            peak, unit, bound, psrc = pk["bf16_tflops"], "TFLOP/s", "tensor", src + ", burst"
        out[name] = {"value": T / (k / 1e3), "unit": "candidates/s", "kernel_ms": k, "steps": n,
                     "dtype": DTYPE[name], "selected_key": d.key,
                     "roofline": {"bound": bound, "achieved": achieved, "peak": peak, "unit": unit,
                                  "frac": achieved / peak, "flop_per_candidate": FLOP_PER_CAND,
                                  "peak_source": psrc},
                     "clocks": cs}
    ab.abacus_load_predictor(ctx, params, PREC[headline])
    torch.cuda.synchronize()
    return out


def whatif_sweep(ab, ctx, slots, H, T, reps=3):
    """NEXT-4 what-if sweep on the config-4 grid: BERT-large's batch size
    swept over {1, 2, 4, 8} (4 x 9.19e9 candidates, abacus_search_whatif).
    Time of the whole blocking call between CUDA events on the current
    stream (the ctx runs on it)."""
    variants = [([8, 8, 8, b], [0, 0, 128, 512]) for b in (1, 2, 4, 8)]
    g = ab.make_grid(slots)
    ab.abacus_search_whatif(ctx, g, variants, H)  # warm-up (grows the buffers)
    import torch
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    kms = []
    for _ in range(reps):
        torch.cuda.synchronize()
        e0.record()
        per, best, bv = ab.abacus_search_whatif(ctx, g, variants, H)
        e1.record()
        torch.cuda.synchronize()
        kms.append(e0.elapsed_time(e1))
    k = float(np.mean(kms))
    n = T * len(variants)
    return {"grid": "config 4, BERT-large bs in {1, 2, 4, 8}", "variants": len(variants), "candidates": n,
            "call_ms": k, "candidates_per_s": n / (k / 1e3), "best_variant": bv, "best_key": best.key,
            "per_variant_total_ops": [d.total_ops for d in per],
            "path": "abacus_search_whatif: 4 variant grids of 9.19e9 candidates (>= 2^24: one fused search "
                    "launch each)"}


def sharded_decision_latency(ab, ctx, comm, world, rank, n=3000, warm=50, label="nccl"):
    """Per-decision latency of abacus_search_sharded on config-3 4-way pure
    GRID decisions (up to 4.1e7 candidates each): every rank searches its
    contiguous shard of each decision's grid and one all-gather combines them
    (SURVEY §8(d)/(e)).  At N = 1 the communicator has one rank.
    Host clock around each blocking call on every rank; the per-decision time
    is the max over ranks."""
    import torch
    import torch.distributed as dist
    decs = synth.cfg3_decisions(n + warm)
    lat = np.zeros(n)
    ev = np.zeros(n)
    for i, (qs, now, infl) in enumerate(decs):
        t0 = time.perf_counter()
        d = ab.abacus_search_sharded(ctx, qs, now, infl, ab.ABACUS_SPACE_GRID, 2**40, comm)
        t1 = time.perf_counter()
        if i >= warm:
            lat[i - warm] = (t1 - t0) * 1e6
            ev[i - warm] = d.evaluated
    t = torch.tensor(lat, dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    a = t.cpu().numpy()
    return {"decisions": n, "n_gpus": world, "space": "grid (pure, config 3, 4-way)",
            "p50_us": float(np.percentile(a, 50)), "p90_us": float(np.percentile(a, 90)),
            "p99_us": float(np.percentile(a, 99)), "p999_us": float(np.percentile(a, 99.9)),
            "max_us": float(a.max()), "grid_p50": float(np.percentile(ev, 50)), "grid_p99": float(np.percentile(ev, 99)),
            "grid_max": float(ev.max()),
            "path": "Python binding -> abacus_search_sharded (%s)" % (
                "NCCL all-gather + finalize kernel over %d rank%s" % (world, "s" if world > 1 else "")
                if label == "nccl" else
                "combine inside the search kernel over %d ranks' peer mailboxes" % world)}


def decision_latency(ab, ctx, n=10_000, warm=100, precision="fp16"):
    """Per-decision latency, host steady clock around each blocking
    abacus_search: (a) through the C ABI (tools/decision_latency.c, no Python
    on the path) for config 2 (3-way GRID) and config 3 (4-way: CHAIN, AUTO
    with two budgets); (b) through the Python binding for config 2."""
    out = {}
    try:
        sys.path.insert(0, os.path.join(ROOT, "tools"))
        import decision_latency as dl
        for cfg, space, budget in (("cfg2", "grid", 0), ("cfg3", "chain", 0), ("cfg3", "auto", 1 << 20),
                                   ("cfg3", "auto", 1 << 22), ("cfg3", "grid", 0)):
            key = "%s_%s" % (cfg, space) + ("_%d" % budget if space == "auto" else "")
            out[key] = dl.run(cfg, space, precision, n, warm, budget or 4_194_304)
        # NEXT-4: many rounds per call (abacus_search_batch), decisions/s
        out["batched"] = {
            "cfg2_grid_b4096": dl.run("cfg2", "grid", precision, 16_384, warm, 4_194_304, batch=4096),
            "cfg3_chain_b4096": dl.run("cfg3", "chain", precision, 16_384, warm, 4_194_304, batch=4096),
            "cfg3_auto_4194304_b1024": dl.run("cfg3", "auto", precision, 4096, warm, 4_194_304, batch=1024),
        }
    except Exception as e:  # noqa: BLE001 -- report, do not fail the bench line
        out["c_abi_error"] = repr(e)
    decs = synth.cfg2_decisions(n + warm)
    lat = []
    for i, (qs, now, infl) in enumerate(decs):
        t0 = time.perf_counter()
        ab.abacus_search(ctx, qs, now, infl, ab.ABACUS_SPACE_GRID)
        t1 = time.perf_counter()
        if i >= warm:
            lat.append((t1 - t0) * 1e6)
    a = np.array(lat)
    out["cfg2_grid_python"] = {"decisions": n, "p50_us": float(np.percentile(a, 50)),
                               "p99_us": float(np.percentile(a, 99)), "p999_us": float(np.percentile(a, 99.9)),
                               "path": "Python binding (ctypes) -> abacus_search"}
    return out


if __name__ == "__main__":
    main()
