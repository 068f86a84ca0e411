for e in 7 8; do timeout 60 python tools/trace_chain.py 100000 engine=$e; done > gpurun_out/exp5.txt 2>&1
timeout 60 python tools/trace_chain.py 100000 engine=8 poll_gap_ns=200 >> gpurun_out/exp5.txt 2>&1
timeout 60 python tools/trace_chain.py 100000 engine=8 backoff_max_ns=32 >> gpurun_out/exp5.txt 2>&1
timeout 60 python tools/trace_chain.py 20000 engine=8 >> gpurun_out/exp5.txt 2>&1
