# compare env-var variants on cfg 3 2 5: usage VARS="KS_FP32_SPLIT=0 KS_FP32_SPLIT=1" bash tools/gpu_variants.sh TAG
TAG=${1:-v}
OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in $VARS; do for c in ${CFGS:-3 2 5}; do
  env $v timeout 600 python bench.py --cfg $c --steps 5 --no-cpu-baseline > $OUT/bench_${v}_cfg$c.json 2>&1
  python - "$OUT/bench_${v}_cfg$c.json" "$v" "$c" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    print(sys.argv[2], "cfg"+sys.argv[3], "value %.4g" % d['value'], "frac %.4f" % d['roofline']['frac'], "kern_ms %.4f" % d['roofline']['kernel_ms'], "clk", d['clocks']['sm_mhz'])
except Exception as e: print(sys.argv[2], sys.argv[3], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done; done
