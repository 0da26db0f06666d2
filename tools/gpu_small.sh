# Small-matrix evidence: copy floors with the band geometry (probe), the 1R1W
# configurations side by side, and the GPU parity tests of the band kernel.
mkdir -p gpurun_out
./tools/probe/geom_copy 4096 s > gpurun_out/small_geom_4k.txt 2>&1
./tools/probe/geom_copy 2048 s > gpurun_out/small_geom_2k.txt 2>&1
python tools/ab_sat.py "4096x4096,3072x3072,2048x2048,1024x1024" "0:0,32:0,16:0,64:0" 10 3 > gpurun_out/small_ab.txt 2>&1
python tools/ab_sat.py "4096x4096,2048x2048" "0:0,32:0,64:0" 10 3 float32 >> gpurun_out/small_ab.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/small_pytest.log 2>&1
