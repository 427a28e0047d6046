# Session-b baseline: cfg1 bench on the current code, then the GEMM rasterisation group swept live (bench, same box)
# and per-GEMM DRAM bytes of one layer under ncu for each group (GEMM DRAM waste).
timeout 900 python bench.py --steps 10 > gpurun_out/r2ba_bench_cfg1.json 2> gpurun_out/r2ba_bench_cfg1.err; echo "bench rc=$?"; head -c 400 gpurun_out/r2ba_bench_cfg1.json; echo
for g in 4 8 32 16; do
  MENOS_GEMM_GROUP_M=$g timeout 600 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/r2ba_bench_g$g.json 2> gpurun_out/r2ba_bench_g$g.err; echo "group $g rc=$?"
  python -c "import json;d=json.load(open('gpurun_out/r2ba_bench_g$g.json'));print('group $g', round(d['value']), d['kernels']['gemm_tcgen05']['ms_per_step'], d['clocks'])"
done
for g in 4 8 16 32; do
  MENOS_GEMM_GROUP_M=$g timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:gemm_tc_kernel -s 24 -c 8 --csv python bench.py --layers 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2ba_gemm_g$g.csv 2> gpurun_out/r2ba_gemm_g$g.err; echo "gemm traffic g$g rc=$?"
done
