timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/torchrun1.json 2> gpurun_out/torchrun1.err; echo tr=$?
tail -c 600 gpurun_out/torchrun1.json; tail -3 gpurun_out/torchrun1.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 1 --steps 1 --warmup 3 > gpurun_out/torchrun1_ref.json 2> gpurun_out/torchrun1_ref.err; echo trref=$?
tail -c 300 gpurun_out/torchrun1_ref.json
