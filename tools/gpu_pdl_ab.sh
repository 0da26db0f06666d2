#!/bin/bash
# A/B of programmatic dependent launch (SAT_PDL) on back-to-back calls and parity with it on.
mkdir -p gpurun_out
for pdl in 0 1; do for n in 1024 4096 16384; do
  SAT_PDL=$pdl timeout 120 python tools/host_overhead.py $n 2>&1 | tail -1 | sed "s/^/pdl=$pdl /"
done; done > gpurun_out/pdl_ab.txt
for pdl in 0 1; do
  SAT_PDL=$pdl timeout 300 python tools/graph_latency.py 2>&1 | sed "s/^/pdl=$pdl /"
done >> gpurun_out/pdl_ab.txt
SAT_PDL=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_box.py -q -x > gpurun_out/pdl_pytest.log 2>&1
echo "pytest exit $?" >> gpurun_out/pdl_pytest.log
