# TC-kernel timing experiments: env variants on the given cfgs (3xtf32)
CF=${CFGS:-3 4}
for v in "$@"; do for c in $CF; do
  env $v python bench.py --cfg $c --precision 3xtf32 --steps ${STEPS:-5} --warmup 2 --no-cpu-baseline 2>&1 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', 'cfg$c', round(d['roofline']['kernel_ms'],3), 'clk', d['clocks']['sm_mhz'])" 2>&1 | tail -1
done; done
