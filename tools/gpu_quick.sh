# quick: gpu tests + bench headline + cfg2/cfg5 + ncu full of fused kernel
TAG=${1:-q}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err
for c in 2 5; do timeout 600 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $OUT/bench_cfg$c.json 2>&1; done
if [ "${NCU:-1}" = "1" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $OUT/prof_cfg3 \
   python bench.py --steps 1 --warmup 4 --no-cpu-baseline > $OUT/ncu_full.log 2>&1
fi
tail -3 $OUT/pytest_gpu.log; tail -1 $OUT/smoke.log
for f in $OUT/bench.json $OUT/bench_cfg2.json $OUT/bench_cfg5.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % d['roofline']['frac'], "kern_ms %.4f" % d['roofline']['kernel_ms'], d['clocks'])
except Exception as e: print(sys.argv[1], "ERR", e, open(sys.argv[1]).read()[-2000:])
PY
done
if [ -n "$VARIANTS" ]; then
for v in $VARIANTS; do for c in 3 2 5; do
  KS_FP32_MINB=$v timeout 600 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $OUT/bench_minb${v}_cfg$c.json 2>&1
  python - "$OUT/bench_minb${v}_cfg$c.json" <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[1], "value %.4g" % d['value'], "frac %.4f" % d['roofline']['frac'], "kern_ms %.4f" % d['roofline']['kernel_ms'], d['config']['ctas'])
PY
done; done
fi
