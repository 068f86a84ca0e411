export PROBE_REPS=10
timeout 600 python tools/probe.py c2,c5,c4 '[{}, {"cta_threads": 256}]' > gpurun_out/exp19_probe.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/exp19_tests.txt 2>&1; echo "rc=$?" >> gpurun_out/exp19_tests.txt
python -c "
import paper_conf_icpp_suz0hw0w20_b200 as cap, numpy as np
for rep in range(3):
    sm, ns = cap.hop_scan(4000, 1)
    thr = 0.5*(np.percentile(ns,5)+np.percentile(ns,95))
    print(rep, round(float(np.median(ns[ns<=thr])),1), round(float(np.median(ns[ns>thr])),1), int((ns<=thr).sum()), int((ns>thr).sum()))
" > gpurun_out/exp19_hop.txt 2>&1
