#!/bin/bash
O=gpurun_out/boxw
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_box.py -x -q > $O/pytest.log 2>&1; echo "exit $?" >> $O/pytest.log
timeout 300 python tools/bench_box.py > $O/box.jsonl 2>&1
timeout 300 python tools/bench_box.py --radius 8 > $O/box_r8.jsonl 2>&1
timeout 300 python tools/bench_box.py --radius 16 > $O/box_r16.jsonl 2>&1
