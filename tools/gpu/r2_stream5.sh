mkdir -p gpurun_out/r7
free -g > gpurun_out/r7/free_before.txt
timeout 1500 python bench.py --config C5 --problems eat --stream-blocks 8 --query-only --k 64 --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/r7/bench_C5_streamed8_k64.json 2> gpurun_out/r7/bench_C5_streamed8_k64.err; echo c5s=$?
free -g > gpurun_out/r7/free_after.txt
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 1 --config C2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r7/bench_C2_torchrun1.json 2> gpurun_out/r7/bench_C2_torchrun1.err; echo tr=$?
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r7/bench_C4.json 2> gpurun_out/r7/bench_C4.err; echo c4=$?
python - <<'PY'
import json
for f in ['bench_C5_streamed8_k64','bench_C2_torchrun1','bench_C4']:
    try:
        d=json.load(open(f'gpurun_out/r7/{f}.json')); r=d['roofline']
        print(f, round(d['value'],2), round(d['ms_per_step'],2), d['rounds'], round(r['frac'],4), (d.get('e2e') or {}).get('value'), d['graph'], d['config'].get('streamed_blocks'))
    except Exception as e: print(f, 'ERR', e)
PY
tail -3 gpurun_out/r7/bench_C5_streamed8_k64.err
