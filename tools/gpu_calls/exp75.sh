timeout 2700 python -m pytest tests -m gpu -q > gpurun_out/exp75_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp75_tests.txt
timeout 1200 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err
timeout 900 python bench.py --impl reference > gpurun_out/bench_ref2.json 2> gpurun_out/bench_ref2.err
rm -rf gpurun_out/r02prof; timeout 1500 bash tools/r02_profile.sh > gpurun_out/r02prof.log 2>&1
