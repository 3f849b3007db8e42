mkdir -p gpurun_out/r3c
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base.so; L=$D/libtempgraph.so; M=$D/libtg_mlp8.so
timeout 900 python tools/job_exp.py C4 1024 $B $L:coarse=0 $L:coarse=1 $M:coarse=1 $B > gpurun_out/r3c/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $B $L:coarse=0 $L:coarse=1 $M:coarse=1 $B > gpurun_out/r3c/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3c/job_*.log
