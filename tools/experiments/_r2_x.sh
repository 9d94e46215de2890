timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "resumed or ladder or usa or c3" > gpurun_out/resume_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/resume_tests.log
timeout 600 python tools/experiments/expand_timeline.py --steps 3 > gpurun_out/expand_timeline_resume.log 2>&1
grep -E "promoted|k_expand" gpurun_out/expand_timeline_resume.log
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 3 --steps 10 > gpurun_out/bench_C3_resume.log 2>&1
python tools/bench_summary.py gpurun_out/bench_C3_resume.log 2>/dev/null || tail -c 600 gpurun_out/bench_C3_resume.log
