mkdir -p gpurun_out/prof2
O=gpurun_out/prof2
KS_EXTRA_NVCC=-DKS_PROF=1 python -m paper_conf_icppw_wangkbgj16_b200.build --force > /dev/null 2>&1
for v in X=0 KS_TC_DEBUG_SKIP_V=10 KS_TC_DEBUG_SKIP_V=1; do
rm -f $O/ctat.txt
env $v KS_CTA_TIMES=$O/ctat.txt python tools/quick_time.py ${CFG:-3} 3 > $O/ctat.log 2>&1
echo "== $v"; python tools/prof_phases.py $O/ctat.txt
done | tee $O/phases.txt
