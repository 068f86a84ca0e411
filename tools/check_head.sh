# HEAD validation on one B200: GPU tests, smoke, the bench line
mkdir -p gpurun_out/head
t0=$(date +%s)
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/head/tests.txt 2>&1; echo "rc=$?" >> gpurun_out/head/tests.txt
t1=$(date +%s)
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/head/smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/head/smoke.txt
timeout 1500 python bench.py > gpurun_out/head/bench.json 2> gpurun_out/head/bench.err; echo "rc=$?" >> gpurun_out/head/bench.err
t2=$(date +%s)
echo "tests $((t1-t0)) s, smoke+bench $((t2-t1)) s" > gpurun_out/head/times.txt
