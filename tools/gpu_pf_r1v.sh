# GEMM epilogue L2 prefetch on/off: isolated dX GEMM timings at cfg1 shapes, then the cfg1 bench; default rebuilt last.
set -x
for v in 1 0; do
  MENOS_NVCC_DEFS="-DMENOS_GEMM_EPI_PREFETCH=$v" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $v"
  timeout 200 python tools/gemm_epi_time.py pf$v >> gpurun_out/pf_r1v.txt 2>&1
  timeout 400 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_r1v_pf$v.json 2>/dev/null; echo "bench v=$v rc=$?"
done
cat gpurun_out/pf_r1v.txt
echo done
