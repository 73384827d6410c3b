#!/bin/bash
# Round-end evidence in one GPU call (run inside gpurun): default bench line, ncu
# launch list of the same command, ncu --set full captures (fused fp16 / bf16,
# predict fp16 / bf16 / fp32 at 2^26 rows, encode / select / encode_groups), HBM
# kernel table, config-5 accuracy, Fig. 23, the reference arm, sanitizers and the
# GPU test suite.  Usage: bash tools/gpu_final.sh <tag>
TAG=${1:-final}
mkdir -p gpurun_out
python -c "import oracle; oracle.build()"
timeout 1200 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-decisions --no-secondary > gpurun_out/${TAG}_launches_bench.json 2>&1
for p in fp16 bf16; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_tc -s 1 -c 1 -o gpurun_out/${TAG}_fused_$p python tools/profile_run.py --precision $p --frac 32 --reps 1 > gpurun_out/${TAG}_ncu_fused_$p.log 2>&1
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:predict24_tc -s 0 -c 1 -o gpurun_out/${TAG}_predict_fp16 python tools/bench_kernels.py --rows 67108864 --reps 1 > gpurun_out/${TAG}_ncu_predict_fp16.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:predict24_tc -s 2 -c 1 -o gpurun_out/${TAG}_predict_bf16 python tools/bench_kernels.py --rows 67108864 --reps 1 > gpurun_out/${TAG}_ncu_predict_bf16.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:predict24_fp32 -s 0 -c 1 -o gpurun_out/${TAG}_predict_fp32 python tools/bench_kernels.py --rows 67108864 --reps 1 > gpurun_out/${TAG}_ncu_predict_fp32.log 2>&1
timeout 600 python tools/bench_kernels.py --out gpurun_out/${TAG}_kernels.json > gpurun_out/${TAG}_kernels.log 2>&1
for k in encode_grid24 select_kernel encode_groups24; do
  timeout 600 ncu --set full --clock-control none -k regex:$k -c 1 -o gpurun_out/${TAG}_$k python tools/bench_kernels.py --rows 16777216 --reps 1 > gpurun_out/${TAG}_ncu_$k.log 2>&1
done
# text summaries on the box; only the top kernel's report comes back whole (gpurun_out <= 64 MiB)
for r in gpurun_out/${TAG}_*.ncu-rep; do
  n=$(basename $r .ncu-rep)
  python tools/ncu_summary.py $r > gpurun_out/${n}_ncu_summary.txt 2>&1
  [ "$n" = "${TAG}_fused_fp16" ] || rm -f $r
done
timeout 900 python tests/accuracy_replay.py --out gpurun_out/${TAG}_cfg5_accuracy.json > gpurun_out/${TAG}_acc.log 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${TAG}_ref.json 2> gpurun_out/${TAG}_ref.err
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_gputests.log 2>&1
echo "pytest exit $?" >> gpurun_out/${TAG}_gputests.log
cat gpurun_out/${TAG}_bench.json | cut -c1-400; tail -3 gpurun_out/${TAG}_bench.err; tail -2 gpurun_out/${TAG}_gputests.log
