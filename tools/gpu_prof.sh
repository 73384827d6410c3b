# ncu --set full of the fused kernel for each exp/<so>:<LINE> entry; summaries + hot list + raw pipe metrics
cd /root/repo
python -c "import oracle; oracle.build()" >/dev/null 2>&1
L=paper_conf_sc_cui0czlzsmylg21_b200/libabacus.so
cp $L /tmp/base.so
for e in "$@"; do
  f=${e%%:*}; ln=${e##*:}
  cp exp/$f.so $L
  ABACUS_LINE=$ln timeout 600 ncu --set full --import-source on --clock-control none -k regex:fused -s 1 -c 1 -o gpurun_out/p_${f}_$ln python tools/profile_run.py --precision fp16 --frac 32 --reps 1 > gpurun_out/p_${f}_$ln.log 2>&1
  python tools/ncu_summary.py gpurun_out/p_${f}_$ln.ncu-rep > gpurun_out/p_${f}_${ln}_summary.txt 2>&1
  python tools/ncu_hot.py gpurun_out/p_${f}_$ln.ncu-rep 80 > gpurun_out/p_${f}_${ln}_hot.txt 2>&1
done
cp /tmp/base.so $L
