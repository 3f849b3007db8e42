mkdir -p gpurun_out/r21
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r21/pytest.log 2>&1; echo pytest=$?
tail -1 gpurun_out/r21/pytest.log
timeout 2000 python tools/job_exp.py C4 1024 $L variants/lib_*.so > gpurun_out/r21/job_C4.log 2>&1
timeout 900 python tools/job_exp.py C2 256 $L variants/lib_*.so > gpurun_out/r21/job_C2.log 2>&1
cat gpurun_out/r21/job_C4.log gpurun_out/r21/job_C2.log | grep "q/s"
