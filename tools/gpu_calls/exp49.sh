export PROBE_REPS=10
for pad in 9000 14000 20000 28000; do
python paper_conf_icpp_suz0hw0w20_b200/build.py -DSPTRSV_MEASURE_HYBRID_SMEM=$pad > /dev/null 2>&1
echo "pad $pad" >> gpurun_out/exp49.txt
(cd tools; timeout 300 python trace_levels.py 1000000 1000 62 >> ../gpurun_out/exp49.txt 2>&1)
timeout 300 python tools/probe.py c4 '[{}]' >> gpurun_out/exp49.txt 2>&1
done
