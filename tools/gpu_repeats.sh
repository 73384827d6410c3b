python -c "import oracle; oracle.build()" >/dev/null 2>&1
for i in 1 2 3; do timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-decisions 2>/dev/null | tail -1 >> gpurun_out/r2j_repeats.jsonl; done
tail -c 300 gpurun_out/r2j_repeats.jsonl
