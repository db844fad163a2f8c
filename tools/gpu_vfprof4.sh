O=gpurun_out/vfprof4; mkdir -p $O
KS_EXTRA_NVCC=-DKS_PROF=1 python -m paper_conf_icppw_wangkbgj16_b200.build --force > $O/build.log 2>&1
rm -f $O/ctat.txt
KS_TC_VCC=0 KS_CTA_TIMES=$O/ctat.txt python tools/quick_time.py 4 1 > $O/ctat.log 2>&1
python tools/prof_phases.py $O/ctat.txt 2>&1
