mkdir -p gpurun_out/fold2
O=gpurun_out/fold2
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -6 $O/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; tail -4 $O/pytest_gpu.log
for c in 3 5; do python tools/quick_time.py $c 10 2>&1 | tail -1 | cut -c1-60; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $O/prof_cfg3 \
   python bench.py --steps 1 --warmup 4 --no-cpu-baseline > $O/ncu_full.log 2>&1
python tools/ncu_summary.py $O/prof_cfg3.ncu-rep > $O/ncu_cfg3.txt 2>&1; head -40 $O/ncu_cfg3.txt
