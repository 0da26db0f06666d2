python tools/ab_sat.py "65536x65536,16384x16384" "128:0:0,128:30:0,128:31:0,128:41:0" 8 2 > gpurun_out/ab4.txt 2>&1
SPECS=$'65536 65536 128 41\n65536 65536 128 0' bash tools/gpu_trace.sh
