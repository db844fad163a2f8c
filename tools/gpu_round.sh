# usage: bash tools/gpu_round.sh TAG  -- tests, bench lines, reference arm, ncu launch list + full captures
TAG=${1:-r01}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > $OUT/nvsmi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 600 python bench.py --precision fp32 --no-cpu-baseline > $OUT/bench_cfg3_fp32.json 2>&1
timeout 600 python bench.py --precision 3xtf32 --no-cpu-baseline > $OUT/bench_cfg3_3xtf32.json 2>&1
for c in 2 5; do timeout 900 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $OUT/bench_cfg$c.json 2>&1; done
for c in 2 5; do timeout 900 python bench.py --cfg $c --steps 5 --precision fp32 --no-cpu-baseline > $OUT/bench_cfg${c}_fp32.json 2>&1; done
timeout 900 python bench.py --cfg 4 --steps 5 --warmup 2 --no-cpu-baseline > $OUT/bench_cfg4.json 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch_bench.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $OUT/prof_cfg3 \
   python bench.py --steps 1 --warmup 4 --no-cpu-baseline > $OUT/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $OUT/prof_cfg3_fp32 \
   python bench.py --precision fp32 --steps 1 --warmup 4 --no-cpu-baseline > $OUT/ncu_full_fp32.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 2 -c 1 -o $OUT/prof_cfg4 \
   python bench.py --cfg 4 --steps 1 --warmup 2 --no-cpu-baseline > $OUT/ncu_full4.log 2>&1
timeout 900 python tools/grid.py $OUT > $OUT/grid.log 2>&1
tail -3 $OUT/pytest_gpu.log; tail -4 $OUT/smoke.log
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    if d.get("impl")=="reference": print(sys.argv[1], "ref value %.4g" % d['value']); raise SystemExit
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % r['frac'], r['bound'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g" % d['e2e']['value'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'])
except SystemExit: pass
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-800:])
PY
done
