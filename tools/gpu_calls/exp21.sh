export PROBE_REPS=10
timeout 900 python tools/probe.py c4 '[{}, {"backoff_max_ns": 0}, {"backoff_max_ns": 16}, {"backoff_min_ns": 0, "backoff_max_ns": 64}, {"warp_split_last": 1}, {"warp_split_last": 0}, {"subwarp": 2}, {"subwarp": 8}, {"subwarp": 1}]' > gpurun_out/exp21_c4.txt 2>&1
timeout 300 python tools/probe.py c2 '[{}, {"backoff_max_ns": 64}, {"backoff_max_ns": 128}, {"backoff_max_ns": 512}, {"poll_one": 1}, {"poll_gap_ns": 32}]' > gpurun_out/exp21_c2.txt 2>&1
