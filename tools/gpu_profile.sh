#!/bin/bash
# round-end style measurement: full default bench, ncu launch list of the same
# command, one ncu --set full capture of the fused kernel and of predict_batch.
TAG=${1:-prof}
python -c "import oracle; oracle.build()"
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-decisions > gpurun_out/${TAG}_launches_bench.json 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_tc -s 1 -c 1 -o gpurun_out/${TAG}_fused_fp16 python tools/profile_run.py --precision fp16 --frac 32 --reps 1 > gpurun_out/${TAG}_ncu_fused.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:predict -s 1 -c 1 -o gpurun_out/${TAG}_predict_fp16 python tools/profile_run.py --precision fp16 --frac 100000 --reps 0 --predict > gpurun_out/${TAG}_ncu_predict.log 2>&1
cat gpurun_out/${TAG}_bench.json; tail -3 gpurun_out/${TAG}_bench.err
