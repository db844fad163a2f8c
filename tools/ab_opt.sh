# A/B of one environment-seeded option through the bench, interleaved on one box:
# bash tools/ab_opt.sh VAR "v1 v2" "cfgs" [reps] [steps]
for rep in $(seq ${4:-2}); do for c in $3; do for v in $2; do
  env $1=$v timeout 300 python bench.py --cfg $c --steps ${5:-20} --no-cpu-baseline --no-traffic --energy-seconds 0.3 2>/dev/null \
   | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('cfg$c $1=$v', round(d['ms_per_step'],4), 'kernel', round(r['kernel_ms'],4), 'clk', round(r.get('kernel_sm_ghz') or 0,3), '%.4e' % d['value'])"
done; done; done
