for o in "engine=8" "engine=8 poll_gap_ns=100" "engine=8 rows_per_lane=2" "engine=8 cta_threads=64 rows_per_lane=2"; do timeout 120 python tools/trace_grid.py 512 $o; done > gpurun_out/exp8_trace.txt 2>&1
timeout 120 python tools/trace_grid.py 512 engine=7 >> gpurun_out/exp8_trace.txt 2>&1
