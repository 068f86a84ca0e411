mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tri.py tests/test_gpu_fuzz.py -x -q -k "lean or tri or fuzz or graph or epoch or solve_host or auto" > gpurun_out/t_lean59.log 2>&1
python tools/optsweep.py c2 '[{}, {"lean_occupancy":5}]' 40 > gpurun_out/sweep59_c2.txt 2>&1
python tools/optsweep.py c5_0 '[{}]' 20 > gpurun_out/sweep59_c5.txt 2>&1
python tools/optsweep.py diag:1000000 '[{}]' 20 > gpurun_out/sweep59_diag.txt 2>&1
