D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $L $D/libtg_v_ubq4.so $L $D/libtg_v_ubq4.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 256 $L $L:ub_filter=2 $D/libtg_v_ubq4.so:ub_filter=2 $L 2>&1 | grep ms
