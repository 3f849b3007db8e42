D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > /tmp/p.log 2>&1; echo pytest=$?; tail -1 /tmp/p.log
timeout 900 python tools/job_exp.py C2 64 $L $L 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 256 $L 2>&1 | grep ms
timeout 900 python tools/job_exp.py C4 64 $L $L 2>&1 | grep ms
timeout 900 python tools/job_exp.py C4 1024 $L 2>&1 | grep ms
timeout 900 python tools/job_exp.py C3 16 $L 2>&1 | grep ms
