# GRID evidence: one --set full capture of k_solve_grid on c3 (the bench config), and the launch list of
# the default bench command (no nested ncu)
mkdir -p gpurun_out/r02grid
ncu --set full --clock-control none --import-source on -k regex:k_solve_grid -s 3 -c 1 -o gpurun_out/r02grid/grid_c3 \
    python tools/run_one.py c3 5 > gpurun_out/r02grid/grid_c3.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/r02grid/launches_bench.csv \
    python bench.py --steps 3 --warmup 3 --no-ncu --no-cpu-baseline > gpurun_out/r02grid/bench_under_ncu.log 2>&1
ls -la gpurun_out/r02grid
