#!/bin/bash
# Every BASELINE config through bench.py (kernel-only lines), plus optional env A/B.
# Logs -> gpurun_out/configs.jsonl
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
: > gpurun_out/configs.jsonl
for cfg in ${CFGS:-cfg1 cfg2 cfg3b cfg3 cfg4 cfg5}; do
  for v in ${VARIANTS_CLI:-1r1w}; do
    env ${ENVS} timeout 300 python bench.py --config $cfg --variant $v --steps ${STEPS:-50} --warmup 5 --no-e2e --no-cpu-baseline \
      >> gpurun_out/configs.jsonl 2>> gpurun_out/configs.log
  done
done
