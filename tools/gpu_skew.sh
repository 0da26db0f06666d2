# build-time A/B: skewed segment-unit ticket order (libsat_skewK.so) vs release
O=gpurun_out
P=$PWD/paper_conf_icpp_kasagini14_b200
LIBSAT_SO=$P/libsat_skew4.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "segments or unit_queue or many" > $O/skew_pytest.log 2>&1
S="65536x65536,32768x32768,24576x24576,20480x20480"
for i in 1 2; do
  python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew_rel_$i.txt 2>&1
  for k in 2 4 8; do LIBSAT_SO=$P/libsat_skew$k.so python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew_${k}_$i.txt 2>&1; done
done
