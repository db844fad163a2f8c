mkdir -p gpurun_out/mbar
O=gpurun_out/mbar
for m in 0 1 2; do
  KS_EXTRA_NVCC="-DKS_MBAR_MODE=$m" python -m paper_conf_icppw_wangkbgj16_b200.build --force > /dev/null 2>&1
  for c in 3 5; do for v in X=0 KS_TC_DEBUG_SKIP_V=10 KS_TC_DEBUG_SKIP_V=1; do
    env $v python tools/quick_time.py $c 10 2>&1 | tail -1 | cut -c1-50 | sed "s/^/MBAR=$m $v: /"
  done; done
done > $O/times.txt 2>&1
cat $O/times.txt
