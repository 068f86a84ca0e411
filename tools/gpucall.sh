mkdir -p gpurun_out
python tools/e2e_probe.py c2 '[{}, {"host_io":2}, {"host_io":0}]' > gpurun_out/e2e71.txt 2>&1
timeout 400 python bench.py --no-cpu-baseline --no-flags-leg --no-tri-leg --nrhs 0 > gpurun_out/bench71.json 2> gpurun_out/bench71.err
timeout 400 python bench.py --no-cpu-baseline --no-flags-leg --no-tri-leg --nrhs 0 > gpurun_out/bench71b.json 2> gpurun_out/bench71b.err
