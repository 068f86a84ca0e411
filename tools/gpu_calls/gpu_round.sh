# full GPU validation: tests, bench (default + N=2 error path), smoke
mkdir -p gpurun_out/r2a
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r2a/tests.txt 2>&1; echo "tests rc=$?" >> gpurun_out/r2a/tests.txt
timeout 900 python bench.py > gpurun_out/r2a/bench.json 2> gpurun_out/r2a/bench.err; echo "bench rc=$?" >> gpurun_out/r2a/bench.err
timeout 300 python bench.py --gpus 2 > gpurun_out/r2a/bench2.json 2> gpurun_out/r2a/bench2.err; echo "bench2 rc=$?" >> gpurun_out/r2a/bench2.err
timeout 300 python bench.py --config c5 > gpurun_out/r2a/bench_c5.json 2> gpurun_out/r2a/bench_c5.err
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2a/smoke.txt 2>&1
