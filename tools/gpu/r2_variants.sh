# EAT relax-kernel tuning variants (query-only CUDA-event timing, C2 EAT+LD and C4 EAT)
for lib in paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so variants/lib_*.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 >> gpurun_out/variants.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/variants.log 2>&1
done
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 9 --launch-count 2 -o gpurun_out/ncu_c2_r2 -f python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/ncu_c2.log 2>&1
echo done
