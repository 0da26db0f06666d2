#!/bin/bash
# Round evidence: bench line, ncu launch list of the bench command, one
# `ncu --set full` capture of the band kernel on the bench workload.
# Outputs -> gpurun_out/ (summarised into profiles/ on the CPU box).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.log
echo "bench exit $?" >> gpurun_out/bench_final.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none -k regex:sat_ --csv --log-file gpurun_out/launches_bench.csv \
  python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sat_band_kernel -s 2 -c 1 \
  -o gpurun_out/prof_cfg4 python tools/prof_one.py cfg4 0 3 > gpurun_out/ncu_full.log 2>&1
for cfg in ${EXTRA_CFGS:-cfg3b}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:sat_band_kernel -s 2 -c 1 \
    -o gpurun_out/prof_$cfg python tools/prof_one.py $cfg 0 3 >> gpurun_out/ncu_full.log 2>&1
done
# export text pages on the box (the .ncu-rep files exceed gpurun's 64 MiB return limit)
for r in gpurun_out/prof_*.ncu-rep; do
  b=${r%.ncu-rep}
  ncu -i $r --page raw --csv > ${b}_raw.csv 2>/dev/null
  ncu -i $r --page details > ${b}_details.txt 2>/dev/null
  ncu -i $r --page source --csv > ${b}_source.csv 2>/dev/null
  rm -f $r
done
