# A/B of the line path (ABACUS_LINE=1) against the layer-1 MMA path, three pairs, plus a short test slice
python -c "import oracle; oracle.build()"
for i in 1 2 3; do for L in 1 0; do
ABACUS_LINE=$L timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-decisions --no-secondary 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('LINE=$L', '%.4e'%d['value'], '%.2f'%d['ms_per_step'], '%.3f'%d['roofline']['frac'], d['selected']['index'], d['selected']['pred_ms'], d['clocks']['sm_mhz'])"
done; done
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -x ${TESTK:+-k "$TESTK"} 2>&1 | tail -15
