mkdir -p gpurun_out/final2
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv > gpurun_out/final2/smi.txt
for c in c2 c1 c3 c4 c5; do timeout 400 python bench.py --config $c > gpurun_out/final2/bench_$c.json 2> gpurun_out/final2/bench_$c.err; done
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final2/ref.json 2> gpurun_out/final2/ref.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final2/launches_c2.csv python bench.py --profile --steps 5 --warmup 3 > gpurun_out/final2/launches_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve_lean --launch-skip 3 -c 1 -o gpurun_out/final2/lean_c2 python bench.py --profile --config c2 --steps 1 --warmup 3 > gpurun_out/final2/ncu_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve_tri_warp --launch-skip 3 -c 1 -o gpurun_out/final2/hybrid_c4 python bench.py --profile --config c4 --steps 1 --warmup 3 > gpurun_out/final2/ncu_c4.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve_chain --launch-skip 3 -c 1 -o gpurun_out/final2/chain_c3 python bench.py --profile --config c3 --steps 1 --warmup 3 > gpurun_out/final2/ncu_c3.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_solve --launch-skip 3 -c 1 -o gpurun_out/final2/oneshot_c1 python bench.py --profile --config c1 --steps 1 --warmup 3 > gpurun_out/final2/ncu_c1.log 2>&1
