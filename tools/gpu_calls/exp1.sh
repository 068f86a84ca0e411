set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
export PROBE_REPS=10
python tools/probe.py c3 '[{}, {"backoff_max_ns": 0}, {"backoff_max_ns": 64}, {"backoff_max_ns": 1024}, {"engine": 3}]' > gpurun_out/exp1_c3.txt 2>&1
python tools/probe.py stride:4194304:2048,stride:1048576:256,chain '[{}, {"backoff_max_ns": 0}, {"backoff_max_ns": 64}, {"engine": 3}]' > gpurun_out/exp1_stride.txt 2>&1
python tools/trace_grid.py 2048 > gpurun_out/exp1_trace.txt 2>&1
python tools/trace_grid.py 2048 backoff_max_ns=0 >> gpurun_out/exp1_trace.txt 2>&1
python tools/trace_grid.py 2048 engine=3 >> gpurun_out/exp1_trace.txt 2>&1
python -c "
import paper_conf_icpp_suz0hw0w20_b200 as cap
for p in range(8):
    print(p, [round(cap.flag_latency(20000, p),1) for _ in range(5)])
" > gpurun_out/exp1_hop.txt 2>&1
