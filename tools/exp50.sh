export PROBE_REPS=10
timeout 600 python tools/probe.py c4 '[{}, {"warp_split_last":3,"poll_gap_ns":0}, {"warp_split_last":3,"poll_gap_ns":50}, {"warp_split_last":3,"poll_gap_ns":100}, {"warp_split_last":3,"poll_gap_ns":200}, {"warp_split_last":3,"poll_gap_ns":400}]' > gpurun_out/exp50.txt 2>&1
(cd tools; timeout 300 python trace_levels.py 1000000 1000 62 warp_split_last=3 poll_gap_ns=100 >> ../gpurun_out/exp50.txt 2>&1)
