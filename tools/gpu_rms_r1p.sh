# RMSNorm d=4096 variants (2 rows x 128 threads, 4 chunks vs 1 row x 256 threads, 2 chunks), isolated timing,
# then the default build's kernel tests, then the split ncu captures of the current code (r1p).
set -x
for v in 0 1; do
  MENOS_NVCC_DEFS="-DMENOS_RMS_WIDE4K=$v" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $v"
  for shp in "8192 4096" "8192 5120" "2048 4096"; do
    echo -n "wide4k=$v " >> gpurun_out/rms_r1p.txt; timeout 120 python tools/rms_time.py $shp >> gpurun_out/rms_r1p.txt 2>&1
  done
  MENOS_NVCC_DEFS="-DMENOS_RMS_WIDE4K=$v" timeout 300 python -m pytest tests/test_gpu_kernels.py -x -q -k rmsnorm > gpurun_out/pytest_rms_r1p_$v.log 2>&1; echo "rms tests v=$v rc=$?"
done
cat gpurun_out/rms_r1p.txt
python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
B="python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1p.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/launches_r1p.log 2>&1; echo "launches rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 40 -c 4 -o gpurun_out/prof_r1p_gemm $B > gpurun_out/ncu_r1p_gemm.log 2>&1; echo "gemm rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 12 -c 2 -o gpurun_out/prof_r1p_abwd $B > gpurun_out/ncu_r1p_abwd.log 2>&1; echo "abwd rc=$?"
timeout 400 ncu --set full --clock-control none -k regex:"rmsnorm|lora_" -s 40 -c 8 -o gpurun_out/prof_r1p_misc $B > gpurun_out/ncu_r1p_misc.log 2>&1; echo "misc rc=$?"
echo done
