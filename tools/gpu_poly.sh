O=gpurun_out/poly; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "host" > $O/pytest_host.log 2>&1; tail -1 $O/pytest_host.log
for r in 1 2; do for pp in 5 6 7; do
  KS_TC_POLY=$pp timeout 300 python bench.py --no-cpu-baseline --steps 30 > $O/bench_pp$pp.json 2>/dev/null
  python - "$O/bench_pp$pp.json" $pp <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
r=d['roofline']; print("PP", sys.argv[2], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g ms %.4f" % (d['e2e']['value'], d['e2e']['ms_per_step']), d['clocks']['sm_mhz'])
PY
done; done
for c in 5 2; do for pp in 5 6 7; do
  KS_TC_POLY=$pp timeout 300 python bench.py --cfg $c --no-cpu-baseline --steps 5 > $O/bench_c${c}_pp$pp.json 2>/dev/null
  python - "$O/bench_c${c}_pp$pp.json" $pp $c <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
r=d['roofline']; print("cfg", sys.argv[3], "PP", sys.argv[2], "value %.4g" % d['value'], "kern_ms %.4f" % r['kernel_ms'], "e2e %.4g" % d['e2e']['value'])
PY
done; done
