# usage: bash tools/gpu_vf.sh TAG -- FP16 V-MMA path: GPU tests (default and forced V-MMA), cfg4 A/B
TAG=${1:-vf}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
KS_TC_VCC=0 timeout 900 python -m pytest tests/test_gpu_tc.py -m gpu -q -x > $OUT/pytest_gpu_vcc0.log 2>&1
tail -3 $OUT/pytest_gpu.log; tail -15 $OUT/pytest_gpu_vcc0.log; tail -6 $OUT/smoke.log
timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4.json 2>&1
KS_TC_VCC=0 timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vf.json 2>&1
KS_TC_VCC=0 KS_TC_AR_STAGES=4 timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vf_ar4.json 2>&1
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % r['frac'], r['bound'], "kern_ms %.4f" % r['kernel_ms'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'], d.get('parity_sampled'))
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done
