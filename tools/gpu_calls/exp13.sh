python -m pytest tests/test_gpu_parity.py -x -q -k "subwarp or hybrid or division_near or solve_host or watchdog or stale or random_small" 2>&1 | tail -5 > gpurun_out/exp13_tests.txt
ABLATION_SET=f2 timeout 1500 python tools/ablation.py 200000 gpurun_out/exp13_f2.jsonl > gpurun_out/exp13_f2.log 2>&1
export PROBE_REPS=10
timeout 600 python tools/probe.py c2,c5,c4 '[{}, {"subwarp": 4, "warp_threshold": 1}, {"subwarp": 2, "warp_threshold": 1}, {"subwarp": 1, "warp_threshold": 1}, {"mode": 3, "subwarp": 4}, {"mode": 3, "subwarp": 8}]' > gpurun_out/exp13_probe.txt 2>&1
