D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $L $L:ub_filter=0 $L $L:ub_filter=0 2>&1 | grep ms
