mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/t_all65.log 2>&1
timeout 1500 python tools/ablation.py 200000 gpurun_out/ablation_final3.jsonl > gpurun_out/ablation_final3.log 2>&1
for c in c1 c2 c3 c4 c5_0 chain; do python tools/optsweep.py $c '[{}]' 10; done > gpurun_out/sweep65.txt 2>&1
