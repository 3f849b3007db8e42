set -x; mkdir -p gpurun_out
for v in "def" "nogc" "slow" "def2"; do
  pre="pass;"; envs=""
  case $v in nogc) pre="import gc; gc.disable();";; slow) envs="BENCH_CLOCK_INTERVAL=0.2";; both) pre="import gc; gc.disable();"; envs="BENCH_CLOCK_INTERVAL=0.2";; esac
  env $envs timeout 300 python -c "$pre import sys, runpy; sys.argv=['bench.py','--steps','20','--warmup','3']; runpy.run_path('bench.py', run_name='__main__')" > gpurun_out/exp_$v.json 2>gpurun_out/exp_$v.err
done
