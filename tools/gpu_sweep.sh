#!/bin/bash
# tile-rows sweep + ncu of the band kernel.  Logs -> gpurun_out/
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for cfg in cfg3b cfg3 cfg4 cfg2 cfg5 cfg1; do
  for th in 16 32 64; do
    timeout 300 python bench.py --config $cfg --tile-rows $th --steps 50 --warmup 5 --no-e2e --no-cpu-baseline \
      >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.log
  done
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sat_band_kernel -s 2 -c 1 \
  -o gpurun_out/prof_cfg3b python tools/prof_one.py cfg3b 0 3 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -s 5 -c 20 --csv \
  --log-file gpurun_out/launches_cfg4.csv python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
