python tools/trace_grid.py 2048 > gpurun_out/exp2_trace.txt 2>&1
python tools/trace_grid.py 2048 rows_per_lane=1 >> gpurun_out/exp2_trace.txt 2>&1
python tools/trace_grid.py 2048 cta_threads=64 >> gpurun_out/exp2_trace.txt 2>&1
python tools/trace_grid.py 2048 cta_threads=256 >> gpurun_out/exp2_trace.txt 2>&1
python tools/trace_grid.py 512 >> gpurun_out/exp2_trace.txt 2>&1
