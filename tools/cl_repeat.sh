#!/bin/bash
# repeat a cluster-path launch in fresh processes; count failures
n=$1; m=$2; reps=$3
fails=0
for i in $(seq 1 $reps); do
  out=$(timeout 60 python tools/cl_probe.py $n $m 2>&1 | grep -E "wrong|failed" | head -1)
  echo "$out" | grep -q "wrong 0" || fails=$((fails+1))
  echo "$i: $out"
done
echo "fails $fails / $reps"
