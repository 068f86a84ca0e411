export PROBE_REPS=5
timeout 300 python tools/probe.py c3,chain '[{}]' > gpurun_out/exp17_probe.txt 2>&1
python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_MEASURE_NO_DIV_PROOF > /dev/null 2>&1
timeout 300 python tools/probe.py c3,chain '[{}]' >> gpurun_out/exp17_probe.txt 2>&1
