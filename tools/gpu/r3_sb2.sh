D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1800 python tools/job_exp.py C4 1024 $L $L:sub_batch=96 $L:sub_batch=128 $L:lanes=2 $L:lanes=3 $L 2>&1 | grep ms
