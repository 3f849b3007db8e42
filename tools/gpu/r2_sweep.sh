mkdir -p gpurun_out/r14
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 2400 python tools/job_exp.py C4 1024 $L variants/lib_*.so > gpurun_out/r14/job_C4.log 2>&1
timeout 900 python tools/job_exp.py C2 256 $L variants/lib_*.so > gpurun_out/r14/job_C2.log 2>&1
cat gpurun_out/r14/job_C4.log gpurun_out/r14/job_C2.log | grep "q/s"
