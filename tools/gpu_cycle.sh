#!/bin/bash
# one GPU iteration: gpu tests, short benches, ncu full capture of the fused kernel
# usage (inside gpurun): bash tools/gpu_cycle.sh <tag> [pytest -k expr]
TAG=${1:-cycle}
K=${2:-}
python -c "import oracle; oracle.build()"
if [ -n "$K" ]; then
  timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -x -k "$K" 2>&1 | tail -25 > gpurun_out/${TAG}_tests.log
else
  timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -x 2>&1 | tail -25 > gpurun_out/${TAG}_tests.log
fi
for p in fp16 bf16 fp32; do
  timeout 600 python bench.py --steps 5 --warmup 3 --precision $p --no-cpu-baseline --no-decisions > gpurun_out/${TAG}_bench_$p.json 2> gpurun_out/${TAG}_bench_$p.err
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused_tc -s 1 -c 1 -o gpurun_out/${TAG}_fused_fp16 python tools/profile_run.py --precision fp16 --frac 32 --reps 1 > gpurun_out/${TAG}_ncu.log 2>&1
cat gpurun_out/${TAG}_tests.log
for p in fp16 bf16 fp32; do python -c "
import json,sys
try:
    d=json.load(open('gpurun_out/${TAG}_bench_$p.json')); print('$p', '%.3e'%d['value'], '%.1f ms'%d['ms_per_step'], 'frac %.3f'%d['roofline']['frac'])
except Exception as e: print('$p', 'FAILED', e); print(open('gpurun_out/${TAG}_bench_$p.err').read()[-2000:])
"; done
