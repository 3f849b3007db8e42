mkdir -p gpurun_out/r3h
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base.so; L=$D/libtempgraph.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3h/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3h/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $B $L $L:ub_filter=0 $B $L > gpurun_out/r3h/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $B $L $L:ub_filter=2 $B $L > gpurun_out/r3h/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3h/job_*.log
