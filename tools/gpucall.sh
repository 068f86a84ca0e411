mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t_all38.log 2>&1
timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/memcheck_small.py > gpurun_out/memcheck38.txt 2>&1; echo "rc=$?" >> gpurun_out/memcheck38.txt
for c in c2 c5; do timeout 400 python bench.py --config $c --no-cpu-baseline --no-flags-leg --no-tri-leg --nrhs 0 > gpurun_out/bench38_$c.json 2> gpurun_out/bench38_$c.err; done
