# One GPU call: OPT (NEXT-4) parity, attention kernels (single-round bwd epilogue, no-RoPE variants), full parity,
# then a cfg1 bench line to measure the attention-backward change.
set -x
timeout 900 python -m pytest tests/test_gpu_opt.py tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_cuts.py tests/test_gpu_serve.py -x -q > gpurun_out/pytest_opt.log 2>&1; echo "pytest rc=$?"
tail -5 gpurun_out/pytest_opt.log
timeout 900 python -m pytest tests/test_gpu_parity_fullsize.py -x -q > gpurun_out/pytest_full.log 2>&1; echo "full rc=$?"
tail -3 gpurun_out/pytest_full.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_cfg1_epi.json 2> gpurun_out/bench_cfg1_epi.err; echo "bench rc=$?"
echo done
