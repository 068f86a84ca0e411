mkdir -p gpurun_out
SPTRSV_FUZZ_SEEDS=600 timeout 1800 python -m pytest tests/test_gpu_fuzz.py -q > gpurun_out/fuzz600.log 2>&1
