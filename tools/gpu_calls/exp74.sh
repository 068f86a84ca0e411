export PROBE_REPS=30
for m in 2 3; do
python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_LEANP_MINB=$m > /dev/null 2>&1 || echo "build fail $m" >> gpurun_out/exp74.txt
echo "minb $m" >> gpurun_out/exp74.txt
timeout 600 python tools/probe.py c2,c5,diag:1000000,lev:1000000:10:4,rand:1000000:3 '[{}, {"engine":3,"mode":1}]' >> gpurun_out/exp74.txt 2>&1
done
