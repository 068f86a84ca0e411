cd tools
for o in "warp_split_last=1 backoff_max_ns=0" "warp_split_last=1 backoff_max_ns=16 backoff_min_ns=0" "warp_split_last=2 backoff_max_ns=0" "warp_split_last=0"; do
timeout 300 python trace_levels.py 1000000 1000 62 $o; done > ../gpurun_out/exp48.txt 2>&1
export PROBE_REPS=20
timeout 300 python probe.py c4 '[{}, {"warp_split_last":1,"backoff_max_ns":0}, {"warp_split_last":2,"backoff_max_ns":0}, {"warp_split_last":1,"backoff_max_ns":16}]' >> ../gpurun_out/exp48.txt 2>&1
