mkdir -p gpurun_out/r4
for lib in paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so variants/lib_nodefer.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 --check >> gpurun_out/r4/variants.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/r4/variants.log 2>&1
done
timeout 900 python tools/order_exp.py C4 1024 > gpurun_out/r4/order_exp.log 2>&1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 1 --mode vertex --exchange 1 --config C2 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r4/bench_C2_vertex_exchange.json 2> gpurun_out/r4/bench_C2_vertex_exchange.err; echo vtx=$?
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r4/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/r4/pytest_gpu.log; grep -h median gpurun_out/r4/variants.log; cat gpurun_out/r4/order_exp.log | grep order; head -c 600 gpurun_out/r4/bench_C2_vertex_exchange.json
