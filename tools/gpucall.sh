mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t_all13.log 2>&1
timeout 400 python bench.py --config c3 --no-cpu-baseline > gpurun_out/bench13_c3.json 2> gpurun_out/bench13_c3.err
python tools/optsweep.py chain '[{}]' 5 > gpurun_out/sweep13_chain.txt 2>&1
