cd /root/repo
for B in 64 256 1024 4096; do python tools/decision_latency.py --config cfg2 --space grid -n 20000 --batch $B; done
for B in 256 1024 4096; do python tools/decision_latency.py --config cfg3 --space auto -n 20000 --batch $B; done
python tools/decision_latency.py --config cfg3 --space chain -n 20000 --batch 4096
python tools/decision_latency.py --config cfg3 --space grid -n 5000 --batch 1024
python tools/decision_latency.py --config cfg2 --space grid -n 20000 --batch 4096 --precision bf16
