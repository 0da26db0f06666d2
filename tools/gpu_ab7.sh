python tools/ab_sat.py "4096x4096,2048x2048,1024x1024,6144x6144,8192x4096" "0:51:0,0:50:0" 10 3 > gpurun_out/ab7.txt 2>&1
python tools/ab_sat.py "4096x4096" "0:51:0,0:50:0" 10 3 float32 >> gpurun_out/ab7.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "cfg1 or cfg2 or shapes or batched or seeded" > gpurun_out/pytest_ab7.log 2>&1
