mkdir -p gpurun_out/r3n
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3n/pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r3n/pytest.log
