# usage: bash tools/gpu_round.sh TAG  -- tests, bench, reference, ncu launch list + full capture of the fused kernel
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > $OUT/nvsmi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch_bench.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $OUT/prof_cfg3 \
   python bench.py --steps 1 --warmup 4 --no-cpu-baseline > $OUT/ncu_full.log 2>&1
for c in 2 5; do timeout 600 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $OUT/bench_cfg$c.json 2>&1; done
tail -3 $OUT/pytest_gpu.log; cat $OUT/smoke.log | tail -2; cat $OUT/bench.json | cut -c1-3000
