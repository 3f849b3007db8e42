mkdir -p gpurun_out/r11
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q -k "insert" > gpurun_out/r11/pytest.log 2>&1; echo pytest=$?
timeout 600 python tools/dynamic_bench.py C2 100000 8 > gpurun_out/r11/dynamic_C2.json 2> gpurun_out/r11/dynamic_C2.err; echo dyn=$?
timeout 900 python tools/dynamic_bench.py C4 100000 4 > gpurun_out/r11/dynamic_C4.json 2> gpurun_out/r11/dynamic_C4.err; echo dyn4=$?
tail -1 gpurun_out/r11/pytest.log; cat gpurun_out/r11/dynamic_C2.json gpurun_out/r11/dynamic_C4.json
