export PROBE_REPS=10
timeout 600 python tools/probe.py c4,lev:100000:1000:6,lev:200000:200:30 '[{}, {"warp_split_k":2}, {"warp_split_k":3}, {"warp_split_k":4}, {"warp_split_k":6}, {"warp_split_k":8}]' > gpurun_out/exp52.txt 2>&1
(cd tools; for k in 1 2 4; do timeout 300 python trace_levels.py 1000000 1000 62 warp_split_k=$k; done >> ../gpurun_out/exp52.txt 2>&1)
