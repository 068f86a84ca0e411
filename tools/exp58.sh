export PROBE_REPS=10
for m in 1 16 20 24 32; do
python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_TRI_WARP_MINB_64=$m > /dev/null 2>&1
echo "minb $m" >> gpurun_out/exp58.txt
timeout 300 python tools/probe.py c4,lev:200000:200:30,lev:100000:1000:6 '[{}]' >> gpurun_out/exp58.txt 2>&1
done
