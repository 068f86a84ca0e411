timeout 600 python bench.py --no-configs --no-ncu --no-e2e --no-tri-leg --nrhs 0 --no-flags-leg > gpurun_out/exp24_bench.json 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/exp24_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp24_tests.txt
