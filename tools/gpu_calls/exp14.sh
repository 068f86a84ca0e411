timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/exp14_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp14_tests.txt
ABLATION_SET=f2 timeout 1500 python tools/ablation.py 200000 gpurun_out/exp14_f2.jsonl > gpurun_out/exp14_f2.log 2>&1
export PROBE_REPS=10
timeout 600 python tools/probe.py c2,c5,c4,c3 '[{}, {"lean_occupancy": 5}]' > gpurun_out/exp14_probe.txt 2>&1
