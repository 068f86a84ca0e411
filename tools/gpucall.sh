mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "solve_host" > gpurun_out/t_host40.log 2>&1
python tools/e2e_probe.py c3 '[{}, {"host_io":0}]' > gpurun_out/e2e40_c3.txt 2>&1
python tools/e2e_probe.py c4 '[{}, {"host_io":0}]' > gpurun_out/e2e40_c4.txt 2>&1
