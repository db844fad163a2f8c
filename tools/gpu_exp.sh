# scratch timing variants: usage CFG=3 bash tools/gpu_exp.sh "ENV=.. prec" ...
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in "$@"; do
  set -- $v
  env $1 python tools/quick_time.py ${CFG:-3} 10 ${2:-auto} 2>&1 | tail -1 | cut -c1-80 | sed "s/^/$1 ${2:-auto}: /"
done
