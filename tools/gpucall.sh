mkdir -p gpurun_out
S='[{"engine":3,"lean_occupancy":5}, {"engine":3,"lean_occupancy":6}, {"engine":3,"lean_occupancy":7}, {"engine":3,"lean_occupancy":8}, {"engine":3,"lean_occupancy":5,"cta_threads":128}, {"engine":3,"lean_occupancy":6,"cta_threads":128}, {"engine":3,"lean_occupancy":7,"cta_threads":128}, {"engine":3,"lean_occupancy":8,"cta_threads":128}, {"engine":3,"lean_occupancy":5,"cta_threads":512}, {"engine":3,"lean_occupancy":6,"cta_threads":512}, {"engine":3,"lean_occupancy":8,"cta_threads":512}, {}]'
python tools/optsweep.py c2 "$S" 20 > gpurun_out/sweep3_c2.txt 2>&1
python tools/optsweep.py c5_0 "$S" 20 > gpurun_out/sweep3_c5.txt 2>&1
python tools/optsweep.py diag:1000000 "$S" 20 > gpurun_out/sweep3_diag.txt 2>&1
python tools/optsweep.py c1 '[{}, {"engine":0,"cta_threads":512}, {"engine":3,"cta_threads":128}]' 30 > gpurun_out/sweep3_c1.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "auto_choice or lean or tri" > gpurun_out/gputests3.log 2>&1
