mkdir -p gpurun_out/r3l
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3l/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3l/pytest.log
for c in C4 C2; do
timeout 900 python tools/build_bench.py $D/libtg_base.so $c --check 2>&1 | tail -3
timeout 900 python tools/build_bench.py $D/libtempgraph.so $c --check 2>&1 | tail -3
done
