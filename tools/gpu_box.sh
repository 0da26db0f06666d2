mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_box.py -x -q > gpurun_out/pytest_box.log 2>&1
python tools/bench_box.py > gpurun_out/box_bench.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:sat_boxf -c 2 --csv --log-file gpurun_out/box_ncu.csv python tools/bench_box.py --reps 1 > /dev/null 2>&1
