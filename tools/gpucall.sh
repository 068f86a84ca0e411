mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_fuzz.py -q > gpurun_out/t_fuzz50.log 2>&1
