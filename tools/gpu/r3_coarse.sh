mkdir -p gpurun_out/r3b
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3b/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/r3b/pytest_gpu.log
timeout 900 python tools/job_exp.py C4 1024 $L:coarse=0 $L:coarse=1 > gpurun_out/r3b/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $L:coarse=0 $L:coarse=1 > gpurun_out/r3b/job_c2.log 2>&1; echo c2=$?
timeout 600 python tools/job_exp.py C1 1 $L:coarse=0 $L:coarse=1 > gpurun_out/r3b/job_c1.log 2>&1; echo c1=$?
cat gpurun_out/r3b/job_*.log
