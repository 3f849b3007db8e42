# usage: bash tools/gpu/variants.sh CFG name1 name2 ...   (libs in variants/)
cfg=$1; shift
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in "$@"; do
  extra=""; [ "$v" != head ] && extra="--check"
  timeout 300 python tools/variant_bench.py variants/lib_$v.so $cfg 64 $extra 2>&1 | grep -v Warning
  [ "$v" == m1b8 -o "$v" == head ] && timeout 300 python tools/variant_bench.py variants/lib_$v.so $cfg 64 --pred 2>&1 | grep -v Warning
done
