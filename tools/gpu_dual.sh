# build-time A/B: two look-backs per control warp (libsat_dual.so) vs release
O=gpurun_out
LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_dual.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not cfg4 and not graph" > $O/dual_pytest.log 2>&1
for i in 1 2; do
  python tools/ab_sat.py "16384x16384,18432x18432,65536x65536,12288x12288" "128:0" 8 2 > $O/dual_rel_$i.txt 2>&1
  LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_dual.so python tools/ab_sat.py "16384x16384,18432x18432,65536x65536,12288x12288" "128:0" 8 2 > $O/dual_on_$i.txt 2>&1
done
