mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "chain or auto_choice" > gpurun_out/t_chain.log 2>&1
python tools/optsweep.py c3 '[{}, {"rows_per_lane":1}, {"backoff_max_ns":512}]' 5 > gpurun_out/sweep10_c3.txt 2>&1
python tools/optsweep.py chain '[{}]' 5 > gpurun_out/sweep10_chain.txt 2>&1
python tools/trace_grid.py 2048 > gpurun_out/trace_grid10.txt 2>&1
