#!/bin/bash
# Final evidence of the round: default bench line, every config, ncu launch
# list + full capture of the band kernel on cfg4 -> gpurun_out/final/
O=gpurun_out/final
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.log
: > $O/configs.jsonl
for cfg in cfg1 cfg2 cfg3b cfg3 cfg4 cfg5; do
  timeout 300 python bench.py --config $cfg --steps 100 --warmup 5 --no-e2e --no-cpu-baseline >> $O/configs.jsonl 2>> $O/configs.log
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none -k regex:sat_ --csv --log-file $O/launches_bench.csv \
  python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/ncu_launch.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sat_band_kernel -s 2 -c 1 \
  -o $O/prof_cfg4 python tools/prof_one.py cfg4 0 3 > $O/ncu_full.log 2>&1
ncu -i $O/prof_cfg4.ncu-rep --page raw --csv > $O/prof_cfg4_raw.csv 2>/dev/null
ncu -i $O/prof_cfg4.ncu-rep --page details > $O/prof_cfg4_details.txt 2>/dev/null
rm -f $O/prof_cfg4.ncu-rep
