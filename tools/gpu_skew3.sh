O=gpurun_out
P=$PWD/paper_conf_icpp_kasagini14_b200
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_float64.py -x -q -k "segments or unit_queue or cfg4 or th128 or batched" > $O/skew3_pytest.log 2>&1
S="65536x65536,49152x49152,32768x32768,24576x24576,20480x20480"
for i in 1 2; do
  LIBSAT_SO=$P/libsat_noskew.so python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew3_old_$i.txt 2>&1
  python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew3_new_$i.txt 2>&1
done
