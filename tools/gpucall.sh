mkdir -p gpurun_out
SPTRSV_FUZZ_SEEDS=400 timeout 1800 python -m pytest tests/test_gpu_fuzz.py -q -k triangular > gpurun_out/fuzz_tri.log 2>&1
timeout 600 python -m pytest tests/test_gpu_fuzz.py -q > gpurun_out/fuzz_default.log 2>&1
