# A/B of exp/*.so variants, default bench, REPS rounds; entries "name:X" (X ignored: the line-path switch of an earlier experiment)
cd /root/repo
python -c "import oracle; oracle.build()" >/dev/null 2>&1
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for rep in $(seq ${REPS:-2}); do
for e in "$@"; do
  f=${e%%:*}; ln=${e##*:}
  cp exp/$f.so $L
  v=$(ABACUS_LINE=$ln timeout 300 python bench.py --steps ${EXP_STEPS:-5} --warmup 3 --no-cpu-baseline --no-decisions --no-secondary 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('%.4e'%d['value'], '%.2f'%d['ms_per_step'], d['selected']['index'], d['selected']['pred_ms'], d['clocks']['sm_mhz'])")
  echo "$f LINE=$ln $v"
done; done
cp /tmp/base.so $L
