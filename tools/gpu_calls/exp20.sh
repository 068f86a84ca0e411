mkdir -p gpurun_out/r02b
timeout 900 python bench.py > gpurun_out/r02b/bench.json 2> gpurun_out/r02b/bench.err
python -c "
import paper_conf_icpp_suz0hw0w20_b200 as cap, numpy as np
for rep in range(2):
    sm, ns = cap.hop_scan(1500, 1)
    thr = 0.5*(np.percentile(ns,5)+np.percentile(ns,95))
    print(rep, round(float(np.median(ns[ns<=thr])),1), round(float(np.median(ns[ns>thr])),1), int((ns<=thr).sum()), int((ns>thr).sum()), np.round(np.percentile(ns,[0,10,50,90,100]),1).tolist())
" > gpurun_out/r02b/hop.txt 2>&1
bash tools/r02_profile.sh > gpurun_out/r02b/profile.log 2>&1
