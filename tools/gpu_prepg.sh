# usage: bash tools/gpu_prepg.sh TAG -- GPU tests + prep-kernel group-size sweep (launch lists + bench)
TAG=${1:-prepg}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
tail -3 $OUT/pytest_gpu.log; tail -6 $OUT/smoke.log
for G in 4 8 16; do
  KS_PREP_G=$G timeout 600 python bench.py --no-cpu-baseline > $OUT/bench_g$G.json 2> $OUT/bench.err
  KS_PREP_G=$G timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file $OUT/launches_g$G.csv \
     python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
  echo "G=$G"; python tools/launch_summary.py $OUT/launches_g$G.csv | head -6
  python - "$OUT/bench_g$G.json" <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % r['frac'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g" % d['e2e']['value'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'])
PY
done
for G in 4 8 32; do
  KS_PREP_G=$G timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file $OUT/launches4_g$G.csv \
     python bench.py --cfg 4 --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
  echo "cfg4 G=$G"; python tools/launch_summary.py $OUT/launches4_g$G.csv | head -6
done
