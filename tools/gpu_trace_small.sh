# Look-back traces of small 1R1W launches (cfg2 geometry, int32 stands in for
# float32: same bytes) with the debug library.  Args: "th:x th:x ..."
mkdir -p gpurun_out
export LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_debug.so
for c in ${1:-32:0}; do
  th=${c%%:*}; x=${c##*:}
  python tools/trace_lookback.py 4096 4096 $th gpurun_out/trace_4k_${th}_$x.npz 0 0 $x > gpurun_out/trace_4k_${th}_$x.log 2>&1
  python tools/analyze_trace.py gpurun_out/trace_4k_${th}_$x.npz >> gpurun_out/trace_4k_${th}_$x.log 2>&1
done
