# One GPU call: 8-warp GEMM epilogue (two warps per TMEM lane quadrant) -- kernel + parity tests, cfg1 bench,
# ncu full set of the GEMMs of one layer (down-dX epilogue-bound before).
set -x
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_opt.py -x -q > gpurun_out/pytest_r1i.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r1i.log
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1i.json 2> gpurun_out/bench_cfg1_r1i.err; echo "bench rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:"gemm_tc_kernel" -s 40 -c 8 -o gpurun_out/prof_r1i python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_r1i.log 2>&1; echo "ncu rc=$?"
echo done
