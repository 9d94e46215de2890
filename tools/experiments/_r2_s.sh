python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 900 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -x -q -k "flush" > gpurun_out/sanitize_flush_r2s.log 2>&1; tail -3 gpurun_out/sanitize_flush_r2s.log
timeout 900 compute-sanitizer --tool racecheck --print-limit 5 python -m pytest tests/test_gpu_parity.py -x -q -k "flush_parity_and_cells and ring" > gpurun_out/racecheck_flush_r2s.log 2>&1; tail -3 gpurun_out/racecheck_flush_r2s.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/gputests_r2s.log 2>&1; tail -3 gpurun_out/gputests_r2s.log
timeout 600 python bench.py > gpurun_out/bench_C3_r2s.log 2>&1; python tools/bench_summary.py gpurun_out/bench_C3_r2s.log
