# usage: bash tools/gpu_pdl.sh TAG -- GPU tests + headline benches with / without programmatic dependent launch
TAG=${1:-pdl}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1
tail -3 $OUT/pytest_gpu.log; tail -8 $OUT/smoke.log
for r in 1 2; do for v in 1 0; do
  KS_PDL=$v timeout 300 python bench.py --no-cpu-baseline --steps 30 > $OUT/bench_pdl${v}_$r.json 2>/dev/null
  KS_PDL=$v timeout 300 python bench.py --cfg 2 --no-cpu-baseline --steps 30 > $OUT/bench_cfg2_pdl${v}_$r.json 2>/dev/null
done; done
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g" % d['e2e']['value'], d['clocks']['sm_mhz'])
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done
