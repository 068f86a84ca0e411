mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tri.py -x -q -k "chain" > gpurun_out/t_chain52.log 2>&1
python tools/optsweep.py c3 '[{}]' 5 > gpurun_out/sweep52_c3.txt 2>&1
python tools/optsweep.py chain '[{}]' 5 > gpurun_out/sweep52_chain.txt 2>&1
python tools/trace_grid.py 2048 > gpurun_out/trace_grid52.txt 2>&1
