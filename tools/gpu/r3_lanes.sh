mkdir -p gpurun_out/r3q
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3q/pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r3q/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $L:lanes=1 $L:lanes=2 $L:lanes=1 $L:lanes=2 > gpurun_out/r3q/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $L:lanes=1 $L:lanes=2 $L:lanes=1 $L:lanes=2 > gpurun_out/r3q/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3q/job_*.log
