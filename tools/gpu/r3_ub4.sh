mkdir -p gpurun_out/r3i
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base.so; L=$D/libtempgraph.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3i/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3i/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $B $L $L:ub_filter=0 $B $L > gpurun_out/r3i/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $B $L $L:ub_filter=2 $B $L > gpurun_out/r3i/job_c2.log 2>&1; echo c2=$?
timeout 600 python tools/job_exp.py C3 16 $B $L $B $L > gpurun_out/r3i/job_c3.log 2>&1; echo c3=$?
cat gpurun_out/r3i/job_*.log
