rm -f gpurun_out/ctat.txt
KS_CTA_TIMES=gpurun_out/ctat.txt python tools/quick_time.py ${1:-3} 3 > gpurun_out/ctat.log 2>&1
python tools/cta_times.py gpurun_out/ctat.txt
