mkdir -p gpurun_out
python tools/optsweep.py c3 '[{}]' 5 > gpurun_out/sweep72_c3.txt 2>&1
python tools/optsweep.py chain '[{}]' 5 > gpurun_out/sweep72_chain.txt 2>&1
python tools/optsweep.py c3 '[{"rows_per_lane":1}]' 5 > gpurun_out/sweep72_c3k1.txt 2>&1
