D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python tools/job_exp.py C4 1024 $D/libtg_v_d32.so $D/libtg_v_d24.so $D/libtg_v_d33.so $D/libtg_v_d32f2.so $D/libtg_v_d32f4.so $D/libtg_v_d32f5.so $D/libtg_v_d32.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 256 $L $D/libtg_v_d24.so $D/libtg_v_d32f4.so $D/libtg_v_d32f5.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 64 $L $D/libtg_v_d32.so $D/libtg_v_d32f4.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C4 128 $L $D/libtg_v_d32.so $D/libtg_v_d32f4.so 2>&1 | grep ms
