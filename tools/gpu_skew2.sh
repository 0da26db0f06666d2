O=gpurun_out
P=$PWD/paper_conf_icpp_kasagini14_b200
S="65536x65536,49152x49152"
for i in 1 2 3; do
  python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew2_rel_$i.txt 2>&1
  for k in 8 16 32; do LIBSAT_SO=$P/libsat_skew$k.so python tools/ab_sat.py "$S" "128:0" 6 2 > $O/skew2_${k}_$i.txt 2>&1; done
done
