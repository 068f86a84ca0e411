mkdir -p gpurun_out
python tools/noticket_probe.py > gpurun_out/noticket58.txt 2>&1
