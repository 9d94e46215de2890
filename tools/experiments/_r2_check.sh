python -m paper_conf_icde_li0qhdy18_b200.build > /dev/null
timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_multi.py -x -q -k "loopback_index_bit_exact and 2" > gpurun_out/sanitize_multi.log 2>&1; tail -3 gpurun_out/sanitize_multi.log
timeout 900 python -m pytest tests/test_gpu_multi.py tests/test_gpu_parity.py -x -q > gpurun_out/gputest_multi_r2b.log 2>&1; tail -3 gpurun_out/gputest_multi_r2b.log
bash tools/run_variants.sh > gpurun_out/variants_r2b.log 2>&1; cat gpurun_out/variants_r2b.log
