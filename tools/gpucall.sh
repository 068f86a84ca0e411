mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "lean_k" > gpurun_out/t_lk.log 2>&1
S='[{}, {"engine":8,"rows_per_lane":2}, {"engine":8,"rows_per_lane":2,"lean_occupancy":3}, {"engine":8,"rows_per_lane":2,"lean_occupancy":5}, {"engine":8,"rows_per_lane":2,"cta_threads":128}, {"engine":8,"rows_per_lane":3}, {"engine":8,"rows_per_lane":3,"lean_occupancy":2}, {"engine":8,"rows_per_lane":4}, {"engine":8,"rows_per_lane":4,"lean_occupancy":3}, {"engine":8,"rows_per_lane":4,"cta_threads":128}]'
python tools/optsweep.py c2 "$S" 20 > gpurun_out/sweep6_c2.txt 2>&1
python tools/optsweep.py c5_0 "$S" 20 > gpurun_out/sweep6_c5.txt 2>&1
python tools/optsweep.py diag:1000000 "$S" 20 > gpurun_out/sweep6_diag.txt 2>&1
python tools/optsweep.py c1 "$S" 20 > gpurun_out/sweep6_c1.txt 2>&1
