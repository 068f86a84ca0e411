mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t_all30.log 2>&1
python tools/optsweep.py c1 '[{}]' 30 > gpurun_out/sweep30_c1.txt 2>&1
