# RMSNorm d=4096 variants: isolated timing, then the cfg1 bench with each (the default build is restored last).
set -x
for v in 0 1; do
  MENOS_NVCC_DEFS="-DMENOS_RMS_WIDE4K=$v" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $v"
  for shp in "8192 4096" "8192 5120" "2048 4096"; do
    echo -n "wide4k=$v " >> gpurun_out/rms_r1q.txt; timeout 120 python tools/rms_time.py $shp >> gpurun_out/rms_r1q.txt 2>&1
  done
  timeout 400 python bench.py --no-cpu-baseline > gpurun_out/bench_r1q_wide$v.json 2> gpurun_out/bench_r1q_wide$v.err; echo "bench v=$v rc=$?"
done
cat gpurun_out/rms_r1q.txt
python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
echo done
