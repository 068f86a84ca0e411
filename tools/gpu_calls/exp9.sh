for o in "engine=8" "engine=8 rows_per_lane=2"; do timeout 120 python tools/trace_grid.py 512 $o; done > gpurun_out/exp9_trace.txt 2>&1
