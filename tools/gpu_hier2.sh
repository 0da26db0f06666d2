#!/bin/bash
# Hierarchical look-back group-size sweep at small sizes.
O=gpurun_out/hier2
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,3072x3072,2048x2048,1024x1024" "0:0:-1,0:0:2,0:0:3,0:0:4,0:0:6" 20 3 float32 > $O/ab_small_f32.txt 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,1024x1024" "0:0:-1,0:0:3,0:0:4" 20 3 int32 > $O/ab_small_i32.txt 2>&1
timeout 600 python tools/ab_sat.py "6144x6144,5120x5120" "0:0:-1,0:0:3,0:0:4,0:0:8" 20 3 int32 > $O/ab_6k.txt 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,2048x2048" "0:0:-1,0:0:3,0:0:4,0:0:8" 20 3 float64 > $O/ab_small_f64.txt 2>&1
