#!/bin/bash
# A/B timing of env knobs: VARIANTS="ENV1=.. ENV2=..;ENV=.." CFGS="cfg3b cfg4"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
out=gpurun_out/ab.txt; : > $out
IFS=';' read -ra VS <<< "${VARIANTS}"
for cfg in ${CFGS:-cfg3b cfg4}; do
  for v in "${VS[@]}"; do
    line=$(env $v timeout 300 python bench.py --config $cfg ${BENCH_EXTRA} --steps ${STEPS:-20} --warmup 3 --no-e2e --no-cpu-baseline 2>>gpurun_out/ab.log)
    echo "$cfg [$v] $(echo "$line" | python -c 'import json,sys; d=json.loads(sys.stdin.read()); r=d["roofline"]; print(r["kernel_ms"], "ms", r["achieved"], "GB/s", "frac", r["frac"], "parity", d["parity_recheck"])')" >> $out
  done
done
cat $out
