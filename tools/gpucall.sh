mkdir -p gpurun_out
python -c "
import ctypes, torch
torch.cuda.init()
lib = ctypes.CDLL('libcudart.so.12') if False else None
print(torch.cuda.get_device_properties(0))
" > gpurun_out/props56.txt 2>&1
python tools/optsweep.py c3 '[{}, {"l2_window":0}]' 5 > gpurun_out/sweep56_c3.txt 2>&1
python tools/optsweep.py c2 '[{}, {"l2_window":0}]' 20 > gpurun_out/sweep56_c2.txt 2>&1
python tools/optsweep.py c4 '[{}]' 10 > gpurun_out/sweep56_c4.txt 2>&1
