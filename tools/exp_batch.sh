# batch-kernel throughput (run inside gpurun): AUTO-4M 1,024-decision and config-2 4,096-decision calls
mkdir -p gpurun_out
python - <<'PY'
import sys, json
sys.path.insert(0, "tools")
import decision_latency as dl
for cfg, space, n, b, bud in (("cfg3", "auto", 4096, 1024, 4194304), ("cfg2", "grid", 16384, 4096, 4194304),
                              ("cfg3", "chain", 16384, 4096, 4194304)):
    r = dl.run(cfg, space, "fp16", n, 100, bud, batch=b)
    print(cfg, space, b, "kernel_us %.1f" % r["kernel_us_mean"], "cand/s(kernel) %.4g" % (r["evaluated_mean"] * b / (r["kernel_us_mean"] * 1e-6)),
          "decisions/s %.4g" % r["decisions_per_s"], flush=True)
PY
