mkdir -p gpurun_out/r9
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
V="$L variants/lib_nodefer.so variants/lib_deg16.so variants/lib_deg32.so variants/lib_deg64.so"
timeout 1500 python tools/job_exp.py C4 1024 $V > gpurun_out/r9/job_C4.log 2>&1
timeout 600 python tools/job_exp.py C2 256 $V > gpurun_out/r9/job_C2.log 2>&1
timeout 600 python tools/job_exp.py C3 64 $V > gpurun_out/r9/job_C3.log 2>&1
timeout 900 python tools/order_exp2.py C4 1024 > gpurun_out/r9/order_exp2.log 2>&1
cat gpurun_out/r9/job_C4.log gpurun_out/r9/job_C2.log gpurun_out/r9/job_C3.log gpurun_out/r9/order_exp2.log | grep "ms"
