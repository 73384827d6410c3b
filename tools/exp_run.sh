#!/bin/bash
# on the GPU box: for each exp/*.so, swap it in and run a short default bench
# (prints cand/s, ms per step and the selected index / pred_ms to spot a wrong variant)
cd /root/repo
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for f in ${@:-exp/*.so}; do
  cp $f $L
  v=$(python bench.py --steps ${EXP_STEPS:-5} --warmup 3 --no-cpu-baseline --no-decisions --no-secondary ${EXP_ARGS} 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.4e'%d['value'], '%.2f'%d['ms_per_step'], d['selected']['index'], d['selected']['pred_ms'])")
  echo "$f $v"
done
cp /tmp/base.so $L
