mkdir -p gpurun_out
for th in 0 16 32 48 64 96 128; do for seg in 1 2 4 8; do
  SAT_SEG=$seg timeout 60 python tools/time_sat.py 4096 4096 float32 $th 30 2>&1 | tail -1 | sed "s/^/seg=$seg th=$th /"
done; done > gpurun_out/cfg2_sweep.txt
for th in 0 16 32 64 128; do for seg in 1 4; do
  SAT_SEG=$seg timeout 60 python tools/time_sat.py 1024 1024 int32 $th 30 2>&1 | tail -1 | sed "s/^/seg=$seg th=$th /"
done; done >> gpurun_out/cfg2_sweep.txt
