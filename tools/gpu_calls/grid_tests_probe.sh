mkdir -p gpurun_out/g1
timeout 900 python -m pytest tests/test_gpu_grid.py -q -x > gpurun_out/g1/t.txt 2>&1
timeout 300 python tools/grid_probe.py c3,g1000,s3d,b1,b8 10 >> gpurun_out/g1/t.txt 2>&1
