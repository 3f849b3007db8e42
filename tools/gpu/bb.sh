# usage: bash tools/gpu/bb.sh CFG name1 name2 ... : build timing of variants (twice) + chain digests
cfg=$1; shift
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do for v in "$@"; do
  timeout 120 python tools/build_bench.py variants/lib_$v.so $cfg --check 2>&1 | grep -v Warn
done; done
