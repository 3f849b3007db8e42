mkdir -p gpurun_out/r3f
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base.so; L=$D/libtempgraph.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3f/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3f/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $B $L:ub_filter=0 $L:ub_filter=1 $B $L:ub_filter=1 > gpurun_out/r3f/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $B $L:ub_filter=0 $L:ub_filter=1 $B $L:ub_filter=1 > gpurun_out/r3f/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3f/job_*.log
