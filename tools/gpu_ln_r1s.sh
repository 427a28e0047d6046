# LayerNorm with 2/4 warps per row for d > 1024: OPT GPU tests, kernel + parity tests, OPT-1.3B paper-setting bench.
set -x
timeout 900 python -m pytest tests/test_gpu_opt.py tests/test_gpu_kernels.py -x -q > gpurun_out/pytest_r1s.log 2>&1; echo "pytest rc=$?"; tail -n 3 gpurun_out/pytest_r1s.log
timeout 400 python bench.py --workload opt13_x16_paper --no-cpu-baseline > gpurun_out/bench_r1s_opt13.json 2> gpurun_out/bench_r1s_opt13.err; echo "bench rc=$?"
echo done
