D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 600 python tools/job_exp.py C2 64 $L $L:sub_batch=32 $L:sub_batch=16 $L 2>&1 | grep ms
timeout 900 python tools/job_exp.py C4 1024 $L $L:sub_batch=32 $L:sub_batch=48 2>&1 | grep ms
timeout 600 python tools/job_exp.py C4 128 $L $L:sub_batch=32 2>&1 | grep ms
