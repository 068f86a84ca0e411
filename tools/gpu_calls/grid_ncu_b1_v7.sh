mkdir -p gpurun_out/g2
timeout 600 ncu --set full --import-source on -k regex:k_solve_grid -s 3 -c 1 -o gpurun_out/g2/grid_b1v7 python tools/grid_probe.py b1 10 > gpurun_out/g2/ncu_b1v7.log 2>&1
