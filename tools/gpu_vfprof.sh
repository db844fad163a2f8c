# usage: bash tools/gpu_vfprof.sh TAG -- ncu full capture of the FP16 V-MMA kernel at cfg4 (+ stage sweep)
TAG=${1:-vfp}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for S in 3 4; do
KS_TC_STAGES=$S KS_TC_VCC=0 timeout 600 python bench.py --cfg 4 --steps 3 --warmup 1 --no-cpu-baseline > $OUT/bench_cfg4_vf_s$S.json 2>&1
done
KS_TC_VCC=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 2 -c 1 -o $OUT/prof_cfg4_vf \
   python bench.py --cfg 4 --steps 1 --warmup 2 --no-cpu-baseline > $OUT/ncu_full4.log 2>&1
for f in $OUT/bench*.json; do python - "$f" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r=d['roofline']; print(sys.argv[1], "value %.4g" % d['value'], "ms %.4f" % d['ms_per_step'], "frac %.4f" % r['frac'], r['bound'], "kern_ms %.4f" % r['kernel_ms'], "clk", d['clocks']['sm_mhz'], d['clocks']['reasons'], d['config'].get('stages'))
except Exception as e: print(sys.argv[1], "ERR", open(sys.argv[1]).read()[-1500:])
PY
done
