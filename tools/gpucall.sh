mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/t_all60.log 2>&1
python tools/optsweep.py c2 '[{}, {"l2_window":0}]' 20 > gpurun_out/sweep60_c2.txt 2>&1
python tools/optsweep.py c4 '[{}]' 10 > gpurun_out/sweep60_c4.txt 2>&1
