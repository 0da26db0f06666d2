#!/bin/bash
# Hierarchical look-back: parity tests, then the A/B of
# group sizes x band heights x sizes behind profiles/r02_hier.txt.
O=gpurun_out/hier
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hier.py -x -q > $O/pytest.log 2>&1; echo "exit $?" >> $O/pytest.log
A="timeout 600 python tools/ab_sat.py"
$A "16384x16384,18432x18432" "128:0:-1,128:0:2,128:0:3,128:0:4,128:0:8,128:0:12,128:0:16,64:0:-1,64:0:4,64:0:8" 10 3 > $O/ab_16k.txt 2>&1
$A "65536x65536" "128:0:-1,128:0:8,128:0:16" 5 2 > $O/ab_64k.txt 2>&1
$A "8192x8192,12288x12288" "0:0:-1,0:0:8,0:0:12" 10 3 > $O/ab_8k.txt 2>&1
$A "6144x6144,5120x5120" "0:0:-1,0:0:3,0:0:4,0:0:8" 20 3 int32 > $O/ab_6k.txt 2>&1
$A "4096x4096,3072x3072,2048x2048,1024x1024" "0:0:-1,0:0:2,0:0:3,0:0:4,0:0:6,16:0:-1,16:0:4" 20 3 float32 > $O/ab_small_f32.txt 2>&1
$A "4096x4096,2048x2048" "0:0:-1,0:0:3,0:0:4,0:0:8" 20 3 float64 > $O/ab_small_f64.txt 2>&1
