mkdir -p gpurun_out/g3
python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_GRID_TRACE > /dev/null 2>&1
timeout 300 python tools/grid_trace.py > gpurun_out/g3/trace2.txt 2>&1
