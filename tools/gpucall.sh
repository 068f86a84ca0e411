mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tri.py -x -q -k "multi or unsupported" > gpurun_out/t_multi42.log 2>&1
