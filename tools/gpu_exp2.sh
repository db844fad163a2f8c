# scratch timing with several env vars per variant: usage CFG=3 bash tools/gpu_exp2.sh "A=1,B=2 prec" ...
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in "$@"; do
  set -- $v
  envs=$(echo $1 | tr ',' ' ')
  env $envs python tools/quick_time.py ${CFG:-3} 10 ${2:-auto} 2>&1 | tail -1 | cut -c1-62 | sed "s/^/$1 ${2:-auto}: /"
done
