mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "solve_host" > gpurun_out/t_host33.log 2>&1
