python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_MEASURE_POLLS -DSPTRSV_MEASURE_ROWSTART > gpurun_out/exp57_build.txt 2>&1
cd tools
timeout 300 python trace_polls.py 1000000 1000 62 > ../gpurun_out/exp57.txt 2>&1
