# build-time A/B: 4 control warps at TH 128 (register cap 96) vs the release library
O=gpurun_out
for i in 1 2; do
  python tools/ab_sat.py "16384x16384,18432x18432,65536x65536" "128:0" 8 2 > $O/ncw_rel_$i.txt 2>&1
  LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_ncw4.so python tools/ab_sat.py "16384x16384,18432x18432,65536x65536" "128:0" 8 2 > $O/ncw_4_$i.txt 2>&1
done
for th in 128 64 32; do timeout 300 python bench.py --config cfg5 --tile-rows $th --steps 100 --no-e2e --no-cpu-baseline >> $O/cfg5_th.jsonl 2>/dev/null; done
