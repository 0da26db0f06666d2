#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/stress.py 4096 4096 3 48 64 > gpurun_out/stress.log 2>&1
python tools/stress.py 16384 4096 3 48 64 >> gpurun_out/stress.log 2>&1
python tools/stress.py 3000 5000 3 48 64 >> gpurun_out/stress.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
for cl in 8 1; do
  rm -f gpurun_out/sweep_cl$cl.jsonl
  for cfg in cfg3b cfg3 cfg4; do
    for th in 48 64; do
      SAT_DEBUG_CL=$cl timeout 300 python bench.py --config $cfg --tile-rows $th --steps 30 --warmup 3 --no-e2e --no-cpu-baseline \
        >> gpurun_out/sweep_cl$cl.jsonl 2>> gpurun_out/sweep.log
    done
  done
done
for th in 64; do
  timeout 120 python tools/trace_lookback.py 16384 16384 $th gpurun_out/trace16k_$th.npz >> gpurun_out/trace.log 2>&1
done
python tools/trace_lookback.py 16384 16384 64 gpurun_out/trace16k_cl.npz >> gpurun_out/trace.log 2>&1
