timeout 2000 python -m pytest tests -m gpu -x -q > gpurun_out/exp15_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp15_tests.txt
export PROBE_REPS=10
timeout 600 python tools/probe.py c3,chain,c2 '[{}]' > gpurun_out/exp15_probe.txt 2>&1
