cd tools
timeout 300 python trace_levels.py 100000 1000 62 > ../gpurun_out/exp51.txt 2>&1
NOFLUSH=1 timeout 300 python trace_levels.py 100000 1000 62 >> ../gpurun_out/exp51.txt 2>&1
timeout 300 python trace_levels.py 100000 1000 6 >> ../gpurun_out/exp51.txt 2>&1
NOFLUSH=1 timeout 300 python trace_levels.py 100000 1000 6 >> ../gpurun_out/exp51.txt 2>&1
timeout 300 python trace_levels.py 1000000 1000 6 >> ../gpurun_out/exp51.txt 2>&1
