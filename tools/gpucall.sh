mkdir -p gpurun_out/final5
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/final5/tests.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final5/smoke.log 2>&1
for c in c2 c1 c3 c4 c5; do timeout 400 python bench.py --config $c > gpurun_out/final5/bench_$c.json 2> gpurun_out/final5/bench_$c.err; done
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final5/ref.json 2> gpurun_out/final5/ref.err
