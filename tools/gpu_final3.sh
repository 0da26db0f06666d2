#!/bin/bash
# End-of-round evidence (round 2, last session) -> gpurun_out/r02g/
O=gpurun_out/r02g
mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/build_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest exit $?" >> $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.log
timeout 600 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.log
: > $O/configs.jsonl
for cfg in cfg1 cfg2 cfg3b cfg3 cfg4 cfg5; do
  timeout 300 python bench.py --config $cfg --steps 100 --warmup 5 --no-e2e --no-cpu-baseline >> $O/configs.jsonl 2>> $O/configs.log
done
for cfg in cfg2 cfg3b; do
  for v in 2r2w 2r1w 1+rr1w 4r4w; do
    timeout 300 python bench.py --config $cfg --variant $v --steps 50 --warmup 5 --no-e2e --no-cpu-baseline >> $O/configs.jsonl 2>> $O/configs.log
  done
done
python tools/bench_box.py > $O/box.jsonl 2>&1
python tools/bench_box.py --radius 8 > $O/box_r8.jsonl 2>&1
timeout 600 python tools/ab_sat.py "4096x4096,6144x6144" "0:0:-1,0:0:0" 20 3 float32 > $O/ab_hier.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none -k regex:sat_ --csv --log-file $O/launches_bench.csv \
  python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > $O/ncu_launch.log 2>&1
for cfg in cfg4 cfg3b cfg2; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sat_band_kernel -s 2 -c 1 \
    -o $O/prof_$cfg python tools/prof_one.py $cfg 0 3 >> $O/ncu_full.log 2>&1
  ncu -i $O/prof_$cfg.ncu-rep --page raw --csv > $O/prof_${cfg}_raw.csv 2>/dev/null
  ncu -i $O/prof_$cfg.ncu-rep --page details > $O/prof_${cfg}_details.txt 2>/dev/null
  rm -f $O/prof_$cfg.ncu-rep
done
timeout 600 ncu --set full --clock-control none -k regex:sat_boxw -s 2 -c 1 -o $O/prof_boxw python tools/prof_box.py 4 >> $O/ncu_full.log 2>&1
ncu -i $O/prof_boxw.ncu-rep --page details > $O/prof_boxw_details.txt 2>/dev/null
ncu -i $O/prof_boxw.ncu-rep --page raw --csv > $O/prof_boxw_raw.csv 2>/dev/null
rm -f $O/prof_boxw.ncu-rep
timeout 400 python tools/fuzz.py --seconds 240 --seed 11 > $O/fuzz11.log 2>&1
