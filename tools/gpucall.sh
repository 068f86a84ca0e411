mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tri.py -x -q -k "lean or tri or hybrid" > gpurun_out/t_lean17.log 2>&1
python tools/optsweep.py c2 '[{}, {"lean_occupancy":5}]' 30 > gpurun_out/sweep17_c2.txt 2>&1
python tools/optsweep.py c5_0 '[{}]' 20 > gpurun_out/sweep17_c5.txt 2>&1
python tools/optsweep.py c4 '[{}]' 10 > gpurun_out/sweep17_c4.txt 2>&1
python tools/optsweep.py diag:1000000 '[{}]' 20 > gpurun_out/sweep17_diag.txt 2>&1
