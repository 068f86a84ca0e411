export PROBE_REPS=5
timeout 600 python tools/probe.py c3,chain,grid:512 '[{"engine": 8, "poll_gap_ns": 32}, {"engine": 8, "poll_gap_ns": 64}, {"engine": 8, "poll_gap_ns": 128}, {"engine": 8, "poll_gap_ns": 256}, {"engine": 8, "poll_gap_ns": 64, "cta_threads": 256}, {"engine": 8, "poll_gap_ns": 64, "backoff_max_ns": 1024}, {"engine": 8, "poll_gap_ns": 128, "backoff_max_ns": 1024}]' > gpurun_out/exp4_probe.txt 2>&1
timeout 120 python tools/trace_grid.py 2048 engine=8 poll_gap_ns=64 > gpurun_out/exp4_trace.txt 2>&1
