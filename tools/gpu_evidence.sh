# Round evidence on one B200 (run through gpurun from the repo root): GPU tests, bench lines for
# every BASELINE config and precision, the reference and unfused arms, the ncu launch list of the
# default bench, ncu --set full captures of the fused kernel per config, compute-sanitizer over the
# newest kernels.  Everything lands in gpurun_out/$TAG; tools/make_profiles.py copies the judged
# parts into profiles/<round>/.  Usage: TAG=r02c bash tools/gpu_evidence.sh [tests|bench|ncu|san]...
set -u
TAG=${TAG:-evidence}
O=gpurun_out/$TAG
mkdir -p $O
parts=${*:-tests bench ncu san}
B="timeout 400 python bench.py"
for p in $parts; do
case $p in
tests)
  timeout 900 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "gpu tests rc=$?" >> $O/gputest.log
  timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1 ;;
bench)
  $B > $O/bench.json 2> $O/bench.err
  $B --cfg 2 --no-cpu-baseline > $O/bench_cfg2.json 2>> $O/bench.err
  $B --cfg 4 --no-cpu-baseline --steps 5 > $O/bench_cfg4.json 2>> $O/bench.err
  $B --cfg 5 --no-cpu-baseline --steps 5 > $O/bench_cfg5.json 2>> $O/bench.err
  for pr in tf32 3xtf32 fp32; do
    $B --precision $pr --no-cpu-baseline --no-traffic > $O/bench_cfg3_$pr.json 2>> $O/bench.err
  done
  $B --impl unfused --no-cpu-baseline > $O/bench_unfused_cfg3.json 2>> $O/bench.err
  $B --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2>> $O/bench.err ;;
ncu)
  ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-traffic --energy-seconds 0 > $O/ncu_launches.log 2>&1
  for c in 3 2 5 4; do
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:ks_fused_ --launch-skip 2 \
      --launch-count 1 -f -o $O/prof_cfg$c python bench.py --traffic-probe --cfg $c > $O/ncu_cfg$c.log 2>&1
  done ;;
san)
  for t in memcheck racecheck synccheck; do
    timeout 900 compute-sanitizer --tool $t --error-exitcode 9 python -m pytest tests/test_gpu_r1.py -q \
      -k "cooperative and (777 or 5000)" > $O/${t}_coop.log 2>&1; echo "rc=$?" >> $O/${t}_coop.log
  done ;;
esac
done
