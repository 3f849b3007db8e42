D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $D/libtg_v_b7.so $D/libtg_v_b8.so $D/libtg_v_b7m2.so $L $D/libtg_v_b7.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 256 $D/libtg_v_b7.so $D/libtg_v_b8.so $D/libtg_v_b7m2.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 64 $L $D/libtg_v_b7.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C1 1 $L $D/libtg_v_b7.so 2>&1 | grep ms
