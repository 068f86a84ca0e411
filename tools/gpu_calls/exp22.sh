export PROBE_REPS=20
timeout 300 python tools/probe.py c1 '[{}, {"backoff_max_ns": 0}, {"backoff_max_ns": 32}, {"local": 0}, {"engine": 3}, {"engine": 7}, {"engine": 6, "mode": 2}, {"cta_threads": 512}, {"backoff_max_ns": 0, "cta_threads": 512}, {"stage_smem": 0}]' > gpurun_out/exp22_c1.txt 2>&1
