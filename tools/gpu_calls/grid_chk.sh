# GRID ring-check granularity: the probe with SPTRSV_GRID_CHK = 8 (per block) / 4 / 2 steps
mkdir -p gpurun_out/chk
for C in 4 2 8; do
  python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_GRID_CHK=$C > gpurun_out/chk/build_$C.txt 2>&1
  timeout 600 python -m pytest tests/test_gpu_grid.py -q -x > gpurun_out/chk/t_$C.txt 2>&1
  timeout 300 python tools/grid_probe.py c3,g1000,s3d,b1,b8 10 > gpurun_out/chk/p_$C.txt 2>&1
done
