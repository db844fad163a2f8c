# phase profile (KS_PROF build) + debug-knob timings of the cfg3 TC kernel
mkdir -p gpurun_out/prof
O=gpurun_out/prof
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in "X=0" "KS_TC_POLY=0" "KS_TC_DEBUG_SKIP_V=5" "KS_TC_DEBUG_SKIP_V=7" "KS_TC_DEBUG_SKIP_V=1"; do
  env $v python tools/quick_time.py ${CFG:-3} 10 2>&1 | tail -1 | cut -c1-70 | sed "s/^/$v: /"
done > $O/knobs.txt
cat $O/knobs.txt
KS_EXTRA_NVCC=-DKS_PROF=1 python -m paper_conf_icppw_wangkbgj16_b200.build --force > /dev/null 2>&1
rm -f $O/ctat.txt
KS_CTA_TIMES=$O/ctat.txt python tools/quick_time.py ${CFG:-3} 3 > $O/ctat.log 2>&1
python tools/prof_phases.py $O/ctat.txt | tee $O/phases.txt
