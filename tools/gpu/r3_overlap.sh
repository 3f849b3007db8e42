mkdir -p gpurun_out/r3p
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 900 python tools/overlap_exp.py C4 512 -1 $D/libtempgraph.so > gpurun_out/r3p/full.log 2>&1; echo a=$?
timeout 900 python tools/overlap_exp.py C4 512 -1 $D/libtg_half.so > gpurun_out/r3p/half.log 2>&1; echo b=$?
timeout 900 python tools/overlap_exp.py C2 256 0 $D/libtg_half.so > gpurun_out/r3p/c2half.log 2>&1; echo c=$?
cat gpurun_out/r3p/*.log
