mkdir -p gpurun_out/final3
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/final3/tests.log 2>&1
for c in c2 c1 c3 c4 c5; do timeout 400 python bench.py --config $c > gpurun_out/final3/bench_$c.json 2> gpurun_out/final3/bench_$c.err; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final3/launches_c2.csv python bench.py --profile --steps 5 --warmup 3 > gpurun_out/final3/launches_c2.log 2>&1
ncu --set full --clock-control none --cache-control none --import-source on -k regex:k_solve_lean --launch-skip 3 -c 1 -o gpurun_out/final3/lean_c2_nocc python bench.py --profile --config c2 --steps 1 --warmup 3 > gpurun_out/final3/ncu_c2.log 2>&1
