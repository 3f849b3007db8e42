mkdir -p gpurun_out/r3x
ncu --metrics gpu__time_duration.sum -c 1 python -c "
import os
print('ENV', {k:v for k,v in os.environ.items() if any(x in k for x in ('INJ','NV_','CUDA','PRELOAD','NSIGHT'))})
import torch; torch.zeros(1, device='cuda')
print('MAPS', [l.split()[-1] for l in open('/proc/self/maps') if 'inject' in l or 'nsight' in l or 'nvperf' in l][:8])
" > gpurun_out/r3x/env.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "lanes or round_loop" > gpurun_out/r3x/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3x/pytest.log
timeout 2400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3x/relax_traffic_C4_job.csv python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/r3x/ncu.log 2>&1; echo ncu=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3x/relax_traffic_C2.csv python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/r3x/ncu2.log 2>&1; echo ncu2=$?
tail -2 gpurun_out/r3x/ncu.log; grep -c gpu__time gpurun_out/r3x/relax_traffic_C4_job.csv; grep -v '^==' gpurun_out/r3x/env.log | head -5
