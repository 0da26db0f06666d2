mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_float64.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_f64.log 2>&1
python tools/ab_sat.py "18432x18432,16384x16384,12288x12288" "128:0,64:0" 8 2 float64 > gpurun_out/ab_f64.txt 2>&1
python tools/ab_sat.py "16384x16384,65536x65536" "128:0" 8 2 int32 >> gpurun_out/ab_f64.txt 2>&1
