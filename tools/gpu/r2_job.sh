mkdir -p gpurun_out/r6
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $L $L:order_sources=0 $L:sub_batch=32 $L:sub_batch=128 variants/lib_nodefer.so variants/lib_defer16.so variants/lib_defer4.so > gpurun_out/r6/job_C4.log 2>&1
timeout 600 python tools/job_exp.py C2 256 $L $L:order_sources=0 $L:sub_batch=32 variants/lib_nodefer.so variants/lib_defer16.so > gpurun_out/r6/job_C2.log 2>&1
cat gpurun_out/r6/job_C4.log gpurun_out/r6/job_C2.log | grep "q/s"
