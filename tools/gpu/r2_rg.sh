mkdir -p gpurun_out/r10
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 600 python tools/job_exp.py C2 64 $L $L:round_group=4 $L:round_group=16 $L:round_group=64 > gpurun_out/r10/rg_C2.log 2>&1
timeout 1500 python tools/job_exp.py C4 1024 $L $L:round_group=16 > gpurun_out/r10/rg_C4.log 2>&1
timeout 600 python tools/job_exp.py C3 16 $L $L:round_group=4 $L:round_group=16 > gpurun_out/r10/rg_C3.log 2>&1
cat gpurun_out/r10/*.log | grep "q/s"
