mkdir -p gpurun_out
python tools/optsweep.py c4 '[{"warp_split_last":2}, {"warp_split_last":3}]' 10 > gpurun_out/sweep45_c4.txt 2>&1
python tools/optsweep.py lev:200000:400 '[{"warp_split_last":2,"mode":2}, {"warp_split_last":3,"mode":2}]' 10 > gpurun_out/sweep45_lev.txt 2>&1
python tools/optsweep.py lev:1000000:1000 '[{"warp_split_last":2,"mode":2}, {"warp_split_last":3,"mode":2}]' 10 > gpurun_out/sweep45_lev2.txt 2>&1
