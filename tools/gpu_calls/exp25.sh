timeout 120 python tools/trace.py c1 > gpurun_out/exp25_c1.txt 2>&1
timeout 120 python tools/trace.py c1 engine=3 >> gpurun_out/exp25_c1.txt 2>&1
