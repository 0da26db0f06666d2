#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/stress.py 4096 4096 5 16 32 48 64 > gpurun_out/stress.log 2>&1; for ns in 1 4; do SAT_DEBUG_CFG=$ns python tools/stress.py 4096 4096 3 32 64 >> gpurun_out/stress.log 2>&1; done
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
rm -f gpurun_out/sweep.jsonl
for cfg in ${CFGS:-cfg3b cfg3 cfg4}; do
  for th in ${THS:-16 32 48 64}; do
    timeout 300 python bench.py --config $cfg --tile-rows $th --steps 30 --warmup 3 --no-e2e --no-cpu-baseline \
      >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.log
  done
done
for th in ${TRACE_THS:-32 64}; do
  timeout 120 python tools/trace_lookback.py 16384 16384 $th gpurun_out/trace16k_$th.npz >> gpurun_out/trace.log 2>&1
done
for ns in ${NS_LIST:-1 4}; do
  rm -f gpurun_out/sweep_ns$ns.jsonl
  for cfg in cfg3b cfg4; do
    for th in 32 64; do
      SAT_DEBUG_CFG=$ns timeout 300 python bench.py --config $cfg --tile-rows $th --steps 30 --warmup 3 --no-e2e --no-cpu-baseline \
        >> gpurun_out/sweep_ns$ns.jsonl 2>> gpurun_out/sweep.log
    done
  done
done
