mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sat_boxf -s 1 -c 1 -o gpurun_out/prof_boxf python tools/bench_box.py --reps 1 > gpurun_out/ncu_boxf.log 2>&1
ncu -i gpurun_out/prof_boxf.ncu-rep --page details > gpurun_out/prof_boxf_details.txt 2>/dev/null
ncu -i gpurun_out/prof_boxf.ncu-rep --page source --csv > gpurun_out/prof_boxf_source.csv 2>/dev/null
ncu -i gpurun_out/prof_boxf.ncu-rep --page raw --csv > gpurun_out/prof_boxf_raw.csv 2>/dev/null
rm -f gpurun_out/prof_boxf.ncu-rep
