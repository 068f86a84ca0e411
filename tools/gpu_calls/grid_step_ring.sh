mkdir -p gpurun_out/g3
B=paper_conf_icpp_suz0hw0w20_b200/build.py
rm -f gpurun_out/g3/sr.txt
for d in "" "-DSPTRSV_GRID_STEP_RING"; do
  python $B --force $d > /dev/null 2>&1
  echo "== $d" >> gpurun_out/g3/sr.txt
  timeout 300 python tools/grid_probe.py c3,g1000,b1 10 >> gpurun_out/g3/sr.txt 2>&1
done
