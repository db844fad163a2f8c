mkdir -p gpurun_out/ares
O=gpurun_out/ares
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -5 $O/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; tail -4 $O/pytest_gpu.log
for c in 3 5 2; do
for v in "X=0" "KS_TC_ARES=0" "KS_TC_POLY=4" "KS_TC_DEBUG_SKIP_V=1"; do
  env $v python tools/quick_time.py $c 10 2>&1 | tail -1 | cut -c1-60 | sed "s/^/$v: /"
done; done > $O/times.txt 2>&1
cat $O/times.txt
