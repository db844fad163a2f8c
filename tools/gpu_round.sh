# One GPU round of evidence (run under gpurun from the repo root): build + smoke, the GPU test
# suite, bench lines (headline + other configs / precisions), the reference arm, the ncu launch
# list of the headline bench and ncu --set full captures of the fused kernel.  Writes
# gpurun_out/$TAG; tools/make_profiles.py copies the judged parts to profiles/<round>.
TAG=${TAG:-round}
O=gpurun_out/$TAG
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -3 $O/smoke.log
if [ "${TESTS:-1}" = "1" ]; then timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; tail -2 $O/pytest_gpu.log; fi
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; tail -c 600 $O/bench.json
for c in ${CFGS:-2 5 4}; do timeout 1200 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $O/bench_cfg$c.json 2> $O/bench_cfg$c.err; done
for p in ${PRECS:-tf32 3xtf32 fp32}; do timeout 900 python bench.py --precision $p --steps 10 --no-cpu-baseline > $O/bench_cfg3_$p.json 2> $O/bench_cfg3_$p.err; done
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2>&1
if [ "${NCU:-1}" = "1" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
     python bench.py --steps 2 --warmup 3 --no-cpu-baseline --energy-seconds 0 > $O/ncu_launches.log 2>&1
  X=sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active,l1tex__data_pipe_tc_wavefronts_mem_shared.sum
  for c in ${NCU_CFGS:-3}; do
    timeout 1200 ncu --set full --metrics $X --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 \
       -o $O/prof_cfg$c python bench.py --cfg $c --steps 1 --warmup 4 --no-cpu-baseline --energy-seconds 0 > $O/ncu_full_cfg$c.log 2>&1
  done
fi
ls $O
