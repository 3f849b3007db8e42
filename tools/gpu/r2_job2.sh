mkdir -p gpurun_out/r6
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $L variants/lib_nodefer.so variants/lib_defer16.so variants/lib_defer4.so > gpurun_out/r6/job_C4b.log 2>&1
grep "q/s" gpurun_out/r6/job_C4b.log; tail -3 gpurun_out/r6/job_C4b.log
