timeout 600 python tools/e2e_probe.py c2 "[{}, {\"engine\":3}]" > gpurun_out/exp78.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tri.py -q -k "solve_host or graph or stale or watchdog or interleav" >> gpurun_out/exp78.txt 2>&1
