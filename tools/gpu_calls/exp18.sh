export PROBE_REPS=5
timeout 300 python tools/probe.py c3,chain '[{}, {"chain_div": 1}]' > gpurun_out/exp18_probe.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/exp18_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp18_tests.txt
