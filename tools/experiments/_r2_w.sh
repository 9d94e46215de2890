GGRID_LIB=$PWD/exp/tail_dbg.so timeout 600 python tools/experiments/expand_timeline.py --steps 3 > gpurun_out/tail_dbg.log 2>&1
grep -c "^P " gpurun_out/tail_dbg.log; tail -5 gpurun_out/tail_dbg.log
