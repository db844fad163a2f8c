mkdir -p gpurun_out/fold
O=gpurun_out/fold
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -6 $O/smoke.log
timeout 900 python -m pytest tests/test_gpu_tc.py -x -q > $O/pytest_tc.log 2>&1; tail -15 $O/pytest_tc.log
for c in 3 5 2; do
for v in "X=0" "KS_TC_POLY=0" "KS_TC_POLY=6" "KS_TC_POLY=8" "KS_TC_FOLD=0"; do
  env $v python tools/quick_time.py $c 10 2>&1 | tail -1 | cut -c1-60 | sed "s/^/$v: /"
done; done > $O/times.txt 2>&1
cat $O/times.txt
