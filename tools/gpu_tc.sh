OUT=gpurun_out/${1:-tc1}; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_tc.py -x -q > $OUT/pytest_tc.log 2>&1; tail -3 $OUT/pytest_tc.log
timeout 600 python bench.py --cfg 4 --steps 5 --warmup 2 --no-cpu-baseline > $OUT/bench_cfg4.json 2>&1
timeout 600 python bench.py --cfg 3 --precision 3xtf32 --steps 10 --no-cpu-baseline > $OUT/bench_cfg3_3xtf32.json 2>&1
timeout 600 python bench.py --cfg 5 --precision 3xtf32 --steps 3 --no-cpu-baseline > $OUT/bench_cfg5_3xtf32.json 2>&1
for f in $OUT/bench_*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.3f" % d['ms_per_step'], "frac %.4f" % r['frac'], "achieved %.1f %s" % (r['achieved'], r['unit'][:20]), "kern_ms %.3f" % r['kernel_ms'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused_tc -s 2 -c 1 -o $OUT/prof_cfg4 \
   python bench.py --cfg 4 --steps 1 --warmup 2 --no-cpu-baseline > $OUT/ncu_full.log 2>&1
tail -1 $OUT/ncu_full.log
