export LIBSAT_SO=$PWD/paper_conf_icpp_kasagini14_b200/libsat_debug.so
python tools/trace_lookback.py 1080 1920 128 gpurun_out/trace_cfg5.npz 0 32 > gpurun_out/trace_cfg5.log 2>&1
