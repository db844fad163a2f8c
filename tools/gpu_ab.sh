# A/B timing on one box: usage bash tools/gpu_ab.sh TAG "cfgs" "env variants..."
TAG=$1; CF=$2; shift 2
mkdir -p gpurun_out/$TAG
O=gpurun_out/$TAG
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -5 $O/smoke.log
if [ "${TESTS:-1}" = "1" ]; then timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; tail -3 $O/pytest_gpu.log; fi
for c in $CF; do
for v in "$@"; do
  env $v python tools/quick_time.py $c 10 2>&1 | tail -1 | cut -c1-60 | sed "s/^/$v: /"
done; done > $O/times.txt 2>&1
cat $O/times.txt
