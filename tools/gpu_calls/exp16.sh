export PROBE_REPS=10
timeout 600 python tools/probe.py c3,chain,c2 '[{}, {"lean_occupancy": 5}, {"lean_occupancy": 5, "cta_threads": 512}, {"lean_occupancy": 5, "cta_threads": 128}]' > gpurun_out/exp16_probe.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "chain or division" > gpurun_out/exp16_tests.txt 2>&1
