export PROBE_REPS=20
timeout 300 python tools/probe.py c1,lev:20000:200:3,lev:4000:40:3 '[{}, {"backoff_max_ns": 32}]' > gpurun_out/exp23_c1.txt 2>&1
python -m pytest tests/test_gpu_parity.py -x -q -k "random_small or c1_config or interleaved or exact_integer" > gpurun_out/exp23_tests.txt 2>&1
