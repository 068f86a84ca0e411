mkdir -p gpurun_out
python tools/optsweep.py c4 '[{"warp_split_last":0}, {"warp_split_last":1}, {"warp_split_last":2}]' 10 > gpurun_out/sweep28_c4.txt 2>&1
python tools/optsweep.py lev:200000:400 '[{"warp_split_last":1,"mode":2}, {"warp_split_last":2,"mode":2}]' 10 > gpurun_out/sweep28_lev.txt 2>&1
