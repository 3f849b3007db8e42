D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 900 python tools/build_bench.py $D/libtg_snapexp.so C4 2>&1 | tail -3
