OUT=gpurun_out/vf3; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 120 ./tools/mma_microbench > $OUT/mma.txt 2>&1; grep -i "unit\|A in" $OUT/mma.txt
KS_TC_VCC=0 KS_TC_DEBUG_SKIP_V=1 timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vf_skipv.json 2>&1
KS_TC_VCC=0 timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vf.json 2>&1
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "kern_ms %.4f" % r['kernel_ms'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done
