# round-2 ncu evidence: launch list of the default bench command (no nested ncu), and one
# --set full capture of each engine's kernel on its config (1 GPU, short commands)
mkdir -p gpurun_out/r02prof
NCU=ncu
$NCU --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/r02prof/launches_bench.csv \
    python bench.py --steps 3 --warmup 3 --no-ncu --no-cpu-baseline > gpurun_out/r02prof/bench_under_ncu.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_solve_lean -s 3 -c 1 -o gpurun_out/r02prof/lean_c2 \
    python tools/run_one.py c2 5 > gpurun_out/r02prof/lean_c2.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_solve_tri_warp -s 3 -c 1 -o gpurun_out/r02prof/hybrid_c4 \
    python tools/run_one.py c4 5 > gpurun_out/r02prof/hybrid_c4.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_solve_chain -s 3 -c 1 -o gpurun_out/r02prof/chain_c3 \
    python tools/run_one.py c3 5 > gpurun_out/r02prof/chain_c3.log 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_solve_small -s 3 -c 1 -o gpurun_out/r02prof/small_c1 \
    python tools/run_one.py c1 5 > gpurun_out/r02prof/small_c1.log 2>&1
ls -la gpurun_out/r02prof
