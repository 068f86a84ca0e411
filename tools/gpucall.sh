mkdir -p gpurun_out/final
for c in c2 c1 c3 c4 c5; do timeout 400 python bench.py --config $c > gpurun_out/final/bench_$c.json 2> gpurun_out/final/bench_$c.err; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final/launches_c2.csv python bench.py --profile --steps 5 --warmup 3 > gpurun_out/final/launches_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve_lean --launch-skip 3 -c 1 -o gpurun_out/final/r01_lean6_c2 python bench.py --profile --config c2 --steps 1 --warmup 3 > gpurun_out/final/ncu_c2.log 2>&1
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final/ref.json 2> gpurun_out/final/ref.err
