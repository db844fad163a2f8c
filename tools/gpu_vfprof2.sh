O=gpurun_out/vfprof; mkdir -p $O
KS_EXTRA_NVCC=-DKS_PROF=1 python -m paper_conf_icppw_wangkbgj16_b200.build --force > $O/build.log 2>&1
for v in "KS_TC_ARES=1" "KS_TC_ARES=0"; do
rm -f $O/ctat.txt
env KS_TC_VCC=0 $v KS_CTA_TIMES=$O/ctat.txt python tools/quick_time.py 4 1 > $O/ctat.log 2>&1
echo "== $v"; python tools/prof_phases.py $O/ctat.txt 2>&1 | head -4
done
