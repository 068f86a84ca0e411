# final round-2 GRID check: GPU suite, smoke, bench, reference arm (tools/final_check.sh), then the ncu
# captures of k_solve_grid (tools/g4.sh) and the bench's launch list
bash tools/final_check.sh
bash tools/g4.sh
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
    --log-file gpurun_out/final/launches.csv python bench.py --steps 2 --warmup 3 > gpurun_out/final/ncu_bench.log 2>&1
