#!/bin/bash
# round-end evidence in one GPU call (run inside gpurun): default bench line,
# ncu launch list of the same command, ncu --set full captures of the fused
# kernel and of predict_batch, HBM kernel table, config-5 accuracy, and a
# short reference-arm (oracle) run.  Usage: bash tools/gpu_final.sh <tag>
TAG=${1:-final}
python -c "import oracle; oracle.build()"
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-decisions > gpurun_out/${TAG}_launches_bench.json 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_tc -s 1 -c 1 -o gpurun_out/${TAG}_fused_fp16 python tools/profile_run.py --precision fp16 --frac 32 --reps 1 > gpurun_out/${TAG}_ncu_fused.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:predict -s 1 -c 1 -o gpurun_out/${TAG}_predict_fp16 python tools/profile_run.py --precision fp16 --frac 100000 --reps 0 --predict > gpurun_out/${TAG}_ncu_predict.log 2>&1
timeout 600 python tools/bench_kernels.py --out gpurun_out/${TAG}_kernels.json > gpurun_out/${TAG}_kernels.log 2>&1
for k in encode_grid24 select_kernel encode_groups24; do
  timeout 600 ncu --set full --clock-control none -k regex:$k -c 1 -o gpurun_out/${TAG}_$k python tools/bench_kernels.py --rows 16777216 --reps 1 > gpurun_out/${TAG}_ncu_$k.log 2>&1
done
timeout 600 python tests/accuracy_replay.py --out gpurun_out/${TAG}_acc.json > gpurun_out/${TAG}_acc.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err
for p in bf16 fp32; do
  timeout 600 python bench.py --steps 5 --warmup 3 --precision $p --no-cpu-baseline --no-decisions > gpurun_out/${TAG}_bench_$p.json 2> gpurun_out/${TAG}_bench_$p.err
done
cat gpurun_out/${TAG}_bench.json | cut -c1-400; tail -3 gpurun_out/${TAG}_bench.err
