# usage: bash tools/gpu_prep.sh TAG -- GPU tests, cfg3 bench, launch list, cfg4 A/B of the V path
TAG=${1:-prep}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_launch_bench.json 2>&1
timeout 900 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4.json 2>&1
KS_TC_VCC=0 timeout 900 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vmma.json 2>&1
tail -3 $OUT/pytest_gpu.log; tail -6 $OUT/smoke.log
python tools/launch_summary.py $OUT/launches.csv | head -12
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % r['frac'], r['bound'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g" % d['e2e']['value'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-800:])
PY
done
