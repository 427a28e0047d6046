# Saved g|u in warp-tile order: epilogue timing, kernel + parity tests and cfg1 bench for EPW = 4 and 8.
set -x
for e in 4 8; do
  MENOS_NVCC_DEFS="-DMENOS_GEMM_EPW=$e" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $e"
  timeout 300 python tools/gemm_epi_time.py tiled_epw$e >> gpurun_out/epi_r1l.jsonl 2>> gpurun_out/epi_r1l.err
  timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_r1l_$e.log 2>&1; echo "pytest $e rc=$?"; tail -2 gpurun_out/pytest_r1l_$e.log
  timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_cfg1_r1l_$e.json 2> gpurun_out/bench_cfg1_r1l_$e.err; echo "bench rc=$?"
done
cat gpurun_out/epi_r1l.jsonl
echo done
