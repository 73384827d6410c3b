# A/B of fused-kernel variants on one box (run inside gpurun): bench lines + parity
mkdir -p gpurun_out
for v in ${VARIANTS:-"4 3 4 3"}; do
  ABACUS_FUSED_RT=$v timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-decisions --no-secondary > gpurun_out/exp_rt$v.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/exp_rt$v.json').read().strip().splitlines()[-1]); print('rt=$v', '%.4g'%d['value'], round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['selected']['key'])"
done
for p in ${PRECS:-bf16}; do
  timeout 300 python bench.py --precision $p --steps 10 --warmup 3 --no-cpu-baseline --no-decisions --no-secondary > gpurun_out/exp_$p.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/exp_$p.json').read().strip().splitlines()[-1]); print('$p', '%.4g'%d['value'], round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['selected']['key'])"
done
[ -n "$NOTEST" ] || timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
