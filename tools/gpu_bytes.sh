O=gpurun_out
for v in 1r1w 2r2w 2r1w 1+rr1w 4r4w; do
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:sat_ --csv --log-file $O/bytes_$v.csv python tools/prof_one.py cfg3b 0 2 $v > /dev/null 2>&1
done
