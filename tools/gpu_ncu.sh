# ncu --set full of the fused kernel for one env variant: usage VAR=... CFG=3 bash tools/gpu_ncu.sh TAG
TAG=${1:-n}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
env ${VAR:-X=1} timeout 900 ncu --set full --clock-control none --import-source on -k regex:ks_fused -s 4 -c 1 -o $OUT/prof_cfg${CFG:-3} \
   python bench.py --cfg ${CFG:-3} --steps 1 --warmup 4 --no-cpu-baseline > $OUT/ncu_full.log 2>&1
tail -2 $OUT/ncu_full.log
