mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/g1_smi.txt
./tools/probe/geom_copy 16384 > gpurun_out/g1_geom16k.txt 2>&1
./tools/probe/geom_copy 65536 > gpurun_out/g1_geom64k.txt 2>&1
timeout 300 python tools/pattern_probe.py 16384 > gpurun_out/g1_pattern.txt 2>&1
