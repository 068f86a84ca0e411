mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_final.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1
