export PROBE_REPS=20
timeout 300 python tools/probe.py c2,c5,diag:1000000 '[{}]' > gpurun_out/exp29_probe.txt 2>&1
