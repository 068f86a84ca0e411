mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/memcheck_small.py > gpurun_out/memcheck18.txt 2>&1; echo "rc=$?" >> gpurun_out/memcheck18.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t_all18.log 2>&1
