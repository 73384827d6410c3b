# A/B of exp/*.so variants on the batched-decision rates (bench.py decision legs)
cd /root/repo
python -c "import oracle; oracle.build()" >/dev/null 2>&1
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for rep in $(seq ${REPS:-2}); do
for f in "$@"; do
  cp exp/$f.so $L
  timeout 600 python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); b=d['decision_latency']['batched']
print('$f', ' '.join('%s %.4g' % (k, v['decisions_per_s']) for k, v in b.items()), 'sweep %.4e' % d['value'])"
done; done
cp /tmp/base.so $L
