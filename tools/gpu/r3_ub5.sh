mkdir -p gpurun_out/r3j
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
B=$D/libtg_base.so; L=$D/libtempgraph.so; Q=$D/libtg_ubq4.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3j/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3j/pytest.log
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 --stats 1 2>&1 | grep diag > gpurun_out/r3j/diag8.log
TG_TRACE=1 timeout 600 python tools/prof_query.py --lib $Q --config C4 --problem eat --k 64 --reps 1 --stats 1 2>&1 | grep diag > gpurun_out/r3j/diag4.log
timeout 900 python tools/job_exp.py C4 1024 $B $L $Q $B $L $Q > gpurun_out/r3j/job_c4.log 2>&1; echo c4=$?
timeout 600 python tools/job_exp.py C2 256 $L:ub_filter=2 $Q:ub_filter=2 $L:ub_filter=0 > gpurun_out/r3j/job_c2.log 2>&1; echo c2=$?
cat gpurun_out/r3j/job_*.log gpurun_out/r3j/diag*.log
