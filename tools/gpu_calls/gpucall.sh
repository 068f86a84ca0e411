mkdir -p gpurun_out
python tools/noticket_probe.py > gpurun_out/noticket76.txt 2>&1
