# One GPU call: kernel + parity tests (fused D epilogue, RMSNorm variants), cfg1 bench, cfg4 TP-8 shard timing, OPT.
set -x
timeout 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_parity_fullsize.py tests/test_gpu_opt.py tests/test_gpu_tp.py -x -q > gpurun_out/pytest_r1g.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r1g.log
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1g.json 2> gpurun_out/bench_cfg1_r1g.err; echo "bench rc=$?"
timeout 900 python bench.py --workload cfg4_70b_tp8_x16 --tp-shard-only 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg4_shard_r1g.json 2> gpurun_out/bench_cfg4_shard_r1g.err; echo "cfg4 rc=$?"
timeout 900 python bench.py --workload opt13_x16_paper --steps 5 --no-cpu-baseline > gpurun_out/bench_opt_r1g.json 2> gpurun_out/bench_opt_r1g.err; echo "opt rc=$?"
echo done
