# GRID evidence: one --set full capture of k_solve_grid on c3 (the bench config)
mkdir -p gpurun_out/r02grid
ncu --set full --clock-control none --import-source on -k regex:k_solve_grid -s 3 -c 1 -o gpurun_out/r02grid/grid_c3_final \
    python tools/run_one.py c3 5 > gpurun_out/r02grid/grid_c3_final.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve_grid -s 3 -c 1 -o gpurun_out/r02grid/grid_b1_final \
    python tools/grid_probe.py b1 10 > gpurun_out/r02grid/grid_b1_final.log 2>&1
