# decision latency A/B over library variants (run inside gpurun): exp_latency.sh lib1.so lib2.so ...
cd /root/repo
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for f in "$@"; do
  cp $f $L
  for cs in "cfg3 chain" "cfg2 grid"; do
    set -- $cs
    r=$(python tools/decision_latency.py --config $1 --space $2 -n 20000 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['p50_us'], d['p99_us'])")
    echo "$f $cs $r"
  done
done
cp /tmp/base.so $L
