#!/bin/bash
# on the GPU box: for each exp/*.so, swap it in and run a short default bench
cd /root/repo
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for f in ${@:-exp/*.so}; do
  cp $f $L
  v=$(python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-decisions 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")
  echo "$f $v"
done
cp /tmp/base.so $L
