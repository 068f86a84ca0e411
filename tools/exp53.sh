python paper_conf_icpp_suz0hw0w20_b200/build.py -DSPTRSV_MEASURE_POLLS > /dev/null 2>&1
cd tools
timeout 300 python trace_polls.py 1000000 1000 62 > ../gpurun_out/exp53.txt 2>&1
timeout 300 python trace_polls.py 100000 1000 6 >> ../gpurun_out/exp53.txt 2>&1
