mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "solve_host or lean" > gpurun_out/t_host24.log 2>&1
timeout 400 python bench.py --config c4 --no-cpu-baseline --no-flags-leg --no-tri-leg --nrhs 0 > gpurun_out/bench24_c4.json 2> gpurun_out/bench24_c4.err
