# FMA-pipe exponential share (option exp_poly, env KS_R1_POLY) per config through the bench, on one
# box, interleaved: prints ms/step, kernel ms and clock.  Usage: bash tools/poly_sweep.sh "5 2" "4 5 6 7 8"
for rep in 1 2; do for c in $1; do for p in $2; do
  KS_R1_POLY=$p timeout 300 python bench.py --cfg $c --steps 8 --no-cpu-baseline --no-traffic --energy-seconds 0.5 2>/dev/null \
   | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; e=d.get('energy',{}); print('cfg$c poly=$p', round(d['ms_per_step'],4), 'kernel', round(r['kernel_ms'],4), 'clk', round(r.get('kernel_sm_ghz') or 0,3), 'J/step', round(e.get('j_per_step',0),4))"
done; done; done
