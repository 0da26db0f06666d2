#!/bin/bash
# Hierarchical look-back: parity tests, then A/B of group sizes.
O=gpurun_out/hier
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hier.py -x -q > $O/pytest.log 2>&1; echo "exit $?" >> $O/pytest.log
timeout 600 python tools/ab_sat.py "16384x16384,18432x18432" "128:0:-1,128:0:4,128:0:8,128:0:12,128:0:16" 10 3 > $O/ab_16k.txt 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,2048x2048" "0:0:-1,0:0:4,0:0:8,0:0:12,0:0:16" 20 3 float32 > $O/ab_4k.txt 2>&1
timeout 600 python tools/ab_sat.py "65536x65536" "128:0:-1,128:0:8,128:0:16" 5 2 > $O/ab_64k.txt 2>&1
timeout 600 python tools/ab_sat.py "8192x8192,12288x12288" "0:0:-1,0:0:8,0:0:12" 10 3 > $O/ab_8k.txt 2>&1
