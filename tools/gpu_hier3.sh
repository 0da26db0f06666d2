#!/bin/bash
# band height x look-back group sweep at small and one-wave sizes
O=gpurun_out/hier3
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,2048x2048,1024x1024" "32:0:-1,32:0:4,16:0:-1,16:0:4,16:0:8" 20 3 float32 > $O/ab_th16.txt 2>&1
timeout 600 python tools/ab_sat.py "16384x16384" "128:0:-1,128:0:2,128:0:3,64:0:-1,64:0:4,64:0:8" 10 3 int32 > $O/ab_16k.txt 2>&1
