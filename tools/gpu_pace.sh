O=gpurun_out
P=$PWD/paper_conf_icpp_kasagini14_b200
LIBSAT_SO=$P/libsat_pace4.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "cfg3 or shapes or jitter or tile_configs" > $O/pace_pytest.log 2>&1
S="16384x16384,18432x18432,12288x12288,8192x8192"
for i in 1 2; do
  python tools/ab_sat.py "$S" "0:0" 8 2 > $O/pace_rel_$i.txt 2>&1
  for d in 2 4 8; do LIBSAT_SO=$P/libsat_pace$d.so python tools/ab_sat.py "$S" "0:0" 8 2 > $O/pace_${d}_$i.txt 2>&1; done
done
