python -m pytest tests/test_gpu_parity.py -x -q -k "chain_engine" 2>&1 | tail -15 > gpurun_out/exp3_tests.txt
export PROBE_REPS=10
timeout 300 python tools/probe.py c3,chain,grid:512 '[{"engine": 7}, {"engine": 8}, {"engine": 8, "rows_per_lane": 1}, {"engine": 8, "cta_threads": 64}, {"engine": 8, "cta_threads": 256}, {"engine": 8, "backoff_max_ns": 64}, {"engine": 8, "backoff_max_ns": 0}]' > gpurun_out/exp3_probe.txt 2>&1
timeout 120 python tools/trace_grid.py 2048 engine=8 > gpurun_out/exp3_trace.txt 2>&1
