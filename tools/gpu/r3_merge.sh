mkdir -p gpurun_out/r3o
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base2.so; L=$D/libtempgraph.so; M16=$D/libtg_m16.so; M1=$D/libtg_m1.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3o/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r3o/pytest.log
timeout 1200 python tools/job_exp.py C4 1024 $B $L $L:merge_big=0 $M16 $M1 $B $L > gpurun_out/r3o/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $B $L $M16 $M1 $B $L > gpurun_out/r3o/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3o/job_*.log
