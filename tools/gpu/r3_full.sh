mkdir -p gpurun_out/r3r
timeout 3000 python -m pytest tests -m gpu -x -q --durations=8 > gpurun_out/r3r/pytest_gpu.log 2>&1; echo pytest=$?; tail -14 gpurun_out/r3r/pytest_gpu.log
