cd tools
timeout 300 python trace_levels.py 1000000 1000 62 > ../gpurun_out/exp47.txt 2>&1
timeout 300 python trace_levels.py 1000000 1000 62 backoff_max_ns=64 >> ../gpurun_out/exp47.txt 2>&1
timeout 300 python trace_levels.py 1000000 1000 62 cta_threads=256 >> ../gpurun_out/exp47.txt 2>&1
timeout 300 python trace_levels.py 200000 1000 62 >> ../gpurun_out/exp47.txt 2>&1
