#!/bin/bash
# GPU test suite + quick bench lines (cfg3b, cfg4 default, cfg2 flushed).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout ${SUITE_TIMEOUT:-1500} python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
for cfg in ${CFGS:-cfg3b cfg2}; do
  timeout 300 python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps ${STEPS:-100} >> gpurun_out/bench_cfgs.jsonl 2>> gpurun_out/bench_cfgs.log
done
