python -m pytest tests/test_gpu_parity.py -x -q -k "subwarp or hybrid or division_near" 2>&1 | tail -5 > gpurun_out/exp12_tests.txt
ABLATION_SET=f2 timeout 1500 python tools/ablation.py 200000 gpurun_out/exp12_f2.jsonl > gpurun_out/exp12_f2.log 2>&1
export PROBE_REPS=10
timeout 300 python tools/probe.py c4 '[{}, {"subwarp": 2}, {"subwarp": 4}, {"subwarp": 8}, {"mode": 3, "subwarp": 4}, {"mode": 3, "subwarp": 2}]' > gpurun_out/exp12_c4.txt 2>&1
