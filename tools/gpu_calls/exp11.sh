python -m pytest tests/test_gpu_parity.py -x -q -k "division or chain_engine or hybrid" 2>&1 | tail -3 > gpurun_out/exp11_tests.txt
export PROBE_REPS=10
timeout 900 python tools/probe.py c4 '[{}, {"warp_split_last": 0}, {"warp_split_last": 1}, {"backoff_max_ns": 32}, {"backoff_max_ns": 64}, {"backoff_max_ns": 1024}, {"backoff_min_ns": 32}, {"mode": 1}, {"warp_threshold": 2}, {"warp_threshold": 20}, {"protocol": 0}, {"l2_window": 0}]' > gpurun_out/exp11_c4.txt 2>&1
