# usage: bash tools/gpu/ab.sh CFG "extra args" name1 name2 ... : alternate variants twice
cfg=$1; shift; extra=$1; shift
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do for v in "$@"; do
  timeout 120 python tools/variant_bench.py variants/lib_$v.so $cfg 64 $extra 2>&1 | grep -v Warn
done; done
