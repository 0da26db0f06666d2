#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
rm -f gpurun_out/sweep_big*.jsonl
for big in 0 1; do
  for cfg in cfg4 cfg3 cfg3b; do
    SAT_BIG=$big timeout 300 python bench.py --config $cfg --tile-rows 64 --steps 30 --warmup 3 --no-e2e --no-cpu-baseline \
      >> gpurun_out/sweep_big$big.jsonl 2>> gpurun_out/sweep.log
  done
done
