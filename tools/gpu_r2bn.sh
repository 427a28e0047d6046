# SwiGLU-bwd epilogue: L2 prefetch of the saved g|u gu_pf chunks beyond the register prefetch (MENOS_GEMM_GU_PF):
# isolated GEMM timing for 0..3, the GEMM kernel tests, and cfg1 bench lines for 0 / 1 / 2 back to back.
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "gemm or swiglu" > gpurun_out/r2bn_gemm_tests.log 2>&1; echo "gemm tests rc=$?"; tail -2 gpurun_out/r2bn_gemm_tests.log
for v in 0 1 2 3; do MENOS_GEMM_GU_PF=$v timeout 300 python tools/gemm_epi_time.py > gpurun_out/r2bn_epi_$v.txt 2>&1; echo "pf $v rc=$?"; grep -i "swiglu_bwd\|down" gpurun_out/r2bn_epi_$v.txt | head -3; done
for v in 0 1 2 0 1 2; do MENOS_GEMM_GU_PF=$v timeout 600 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/r2bn_bench_$v.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/r2bn_bench_$v.json'));print('pf $v', round(d['value']), round(d['kernels']['gemm_tcgen05']['ms_per_step'],2), d['clocks']['sm_mhz'])"; done
