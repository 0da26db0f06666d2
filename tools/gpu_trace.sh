#!/bin/bash
# Look-back event traces (debug build) of one 1R1W launch per spec line
# "rows cols tile_rows segments" (SPECS, newline-separated).
mkdir -p gpurun_out
export LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_debug.so
SPECS=${SPECS:-$'16384 16384 128 0\n65536 65536 128 0'}
while read -r r c th x; do
  [ -z "$r" ] && continue
  python tools/trace_lookback.py $r $c $th gpurun_out/trace_${r}_${th}_${x}.npz $x > gpurun_out/trace_${r}_${th}_${x}.log 2>&1
done <<< "$SPECS"
