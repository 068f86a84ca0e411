mkdir -p gpurun_out
python tools/trace.py c1 > gpurun_out/trace_c1_39.txt 2>&1
timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tests/memcheck_driver.py > gpurun_out/memcheck39.txt 2>&1; echo "rc=$?" >> gpurun_out/memcheck39.txt
