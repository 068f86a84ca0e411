python -m pytest tests/test_gpu_parity.py -x -q -k "chain_engine or hybrid_engine" 2>&1 | tail -5 > gpurun_out/exp6_tests.txt
export PROBE_REPS=5
timeout 600 python tools/probe.py c3,chain,grid:512 '[{"engine": 8}, {"engine": 8, "rows_per_lane": 4}, {"engine": 8, "rows_per_lane": 2}, {"engine": 8, "cta_threads": 64}, {"engine": 8, "cta_threads": 256}, {"engine": 8, "backoff_max_ns": 64}, {"engine": 8, "poll_gap_ns": 64}]' > gpurun_out/exp6_probe.txt 2>&1
timeout 120 python tools/trace_grid.py 2048 engine=8 > gpurun_out/exp6_trace.txt 2>&1
timeout 60 python tools/trace_chain.py 100000 engine=8 >> gpurun_out/exp6_trace.txt 2>&1
python -c "
import paper_conf_icpp_suz0hw0w20_b200 as cap, numpy as np
for pr in (1, 0):
  for rep in range(2):
    sm, ns = cap.hop_scan(4000, pr)
    print(pr, len(sm), np.round(np.percentile(ns,[0,5,25,50,75,95,100]),1).tolist())
    print(' '.join('%d:%.0f'%(a,b) for a,b in zip(sm,ns)))
" > gpurun_out/exp6_hop.txt 2>&1
