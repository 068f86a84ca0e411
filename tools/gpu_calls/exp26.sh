mkdir -p gpurun_out/r02c
timeout 900 python bench.py > gpurun_out/r02c/bench.json 2> gpurun_out/r02c/bench.err
timeout 300 python bench.py --impl reference > gpurun_out/r02c/ref.json 2> gpurun_out/r02c/ref.err
timeout 300 python bench.py --gpus 2 > gpurun_out/r02c/bench2.json 2> gpurun_out/r02c/bench2.err; echo "rc=$?" >> gpurun_out/r02c/bench2.err
timeout 300 python bench.py --config c5 > gpurun_out/r02c/bench_c5.json 2> gpurun_out/r02c/bench_c5.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02c/smoke.txt 2>&1
