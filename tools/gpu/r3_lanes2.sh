mkdir -p gpurun_out/r3s
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3s/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r3s/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $L:lanes=1 $L:lanes=2 $L:lanes=3 $L:lanes=4 $L:lanes=2 > gpurun_out/r3s/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $L:lanes=1 $L:lanes=2 $L:lanes=3 $L:lanes=4 $L:lanes=2 > gpurun_out/r3s/job_c2.log 2>&1; echo c2=$?
timeout 600 python tools/job_exp.py C2 1024 $L:lanes=2 $L:lanes=4 > gpurun_out/r3s/job_c2b.log 2>&1
cat gpurun_out/r3s/job_*.log
