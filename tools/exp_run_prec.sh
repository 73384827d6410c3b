#!/bin/bash
# on the GPU box: like exp_run.sh, for a given precision: exp_run_prec.sh <fp32|fp16|bf16> lib.so ...
cd /root/repo
P=$1; shift
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for f in "$@"; do
  cp $f $L
  v=$(python bench.py --precision $P --steps ${EXP_STEPS:-3} --warmup 3 --no-cpu-baseline --no-decisions 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.4e'%d['value'], '%.2f'%d['ms_per_step'], d['selected']['index'], d['selected']['pred_ms'])")
  echo "$P $f $v"
done
cp /tmp/base.so $L
