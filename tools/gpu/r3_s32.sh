D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 900 python tools/job_exp.py C2 64 $L $D/libtg_v_s32.so $D/libtg_v_s32d8.so $L $D/libtg_v_s32.so $D/libtg_v_s32d8.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C4 64 $L $D/libtg_v_s32.so $L $D/libtg_v_s32.so 2>&1 | grep ms
