# round-2 validation on one B200: GPU tests, smoke, the bench line (timed), the reference arm
mkdir -p gpurun_out/final
t0=$(date +%s)
timeout 2700 python -m pytest tests -m gpu -q > gpurun_out/final/tests.txt 2>&1; echo "rc=$?" >> gpurun_out/final/tests.txt
t1=$(date +%s)
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.txt 2>&1; echo "rc=$?" >> gpurun_out/final/smoke.txt
t2=$(date +%s)
timeout 1500 python bench.py > gpurun_out/final/bench.json 2> gpurun_out/final/bench.err; echo "rc=$?" >> gpurun_out/final/bench.err
t3=$(date +%s)
timeout 900 python bench.py --impl reference > gpurun_out/final/ref.json 2> gpurun_out/final/ref.err; echo "rc=$?" >> gpurun_out/final/ref.err
t4=$(date +%s)
echo "tests $((t1-t0)) s, smoke $((t2-t1)) s, bench $((t3-t2)) s, reference $((t4-t3)) s" > gpurun_out/final/times.txt
