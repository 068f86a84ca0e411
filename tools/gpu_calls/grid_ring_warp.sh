mkdir -p gpurun_out/g3
B=paper_conf_icpp_suz0hw0w20_b200/build.py
rm -f gpurun_out/g3/rw.txt
for d in "-DSPTRSV_GRID_RING_WARP=5" "-DSPTRSV_GRID_RING_WARP=4"; do
  python $B --force $d > /dev/null 2>&1
  echo "== $d" >> gpurun_out/g3/rw.txt
  timeout 300 python tools/grid_probe.py c3,g1000,b1,b8 10 >> gpurun_out/g3/rw.txt 2>&1
done
timeout 600 python -m pytest tests/test_gpu_grid.py -q -x >> gpurun_out/g3/rw.txt 2>&1
