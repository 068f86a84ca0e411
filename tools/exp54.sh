python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_MEASURE_POLLS > /dev/null 2>&1
cd tools
timeout 300 python trace_polls.py 1000000 1000 62 > ../gpurun_out/exp54.txt 2>&1
timeout 300 python trace_polls.py 100000 1000 6 >> ../gpurun_out/exp54.txt 2>&1
cd ..
export PROBE_REPS=10
for pad in 0 9000 14000 28000; do
if [ $pad = 0 ]; then python paper_conf_icpp_suz0hw0w20_b200/build.py --force > /dev/null 2>&1; else python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_MEASURE_HYBRID_SMEM=$pad > /dev/null 2>&1; fi
echo "pad $pad" >> gpurun_out/exp54.txt
(cd tools; timeout 300 python trace_levels.py 1000000 1000 62 >> ../gpurun_out/exp54.txt 2>&1)
timeout 300 python tools/probe.py c4 '[{}]' >> gpurun_out/exp54.txt 2>&1
done
