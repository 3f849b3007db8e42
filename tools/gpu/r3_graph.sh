mkdir -p gpurun_out/r3m
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3m/pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r3m/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $L:graph_loop=0 $L:graph_loop=1 $L:graph_loop=0 $L:graph_loop=1 > gpurun_out/r3m/job_c4.log 2>&1; echo c4=$?
for c in "C2 256" "C2 64" "C3 16" "C1 1"; do timeout 600 python tools/job_exp.py $c $L:graph_loop=0 $L:graph_loop=1 $L:graph_loop=0 $L:graph_loop=1 >> gpurun_out/r3m/job_small.log 2>&1; done; echo small=$?
cat gpurun_out/r3m/job_*.log
