python -m pytest tests/test_gpu_parity.py -x -q -k "chain_engine or hybrid_engine" 2>&1 | tail -3 > gpurun_out/exp7_tests.txt
export PROBE_REPS=5
timeout 600 python tools/probe.py c3,chain,grid:512 '[{"engine": 8}, {"engine": 8, "rows_per_lane": 4}, {"engine": 8, "cta_threads": 64}, {"engine": 8, "backoff_max_ns": 64}]' > gpurun_out/exp7_probe.txt 2>&1
timeout 120 python tools/trace_grid.py 2048 engine=8 > gpurun_out/exp7_trace.txt 2>&1
timeout 60 python tools/trace_chain.py 100000 engine=8 >> gpurun_out/exp7_trace.txt 2>&1
