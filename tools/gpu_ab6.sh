python tools/ab_sat.py "65536x65536,16384x16384,18432x18432" "128:0:0,128:41:0" 8 2 > gpurun_out/ab6.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_float64.py tests/test_gpu_box.py -x -q > gpurun_out/pytest_ab6.log 2>&1
for cfg in cfg5 cfg2 cfg1; do timeout 300 python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps 200 >> gpurun_out/ab6_bench.jsonl 2>/dev/null; done
