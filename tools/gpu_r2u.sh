# Attention-backward epilogue rework (RoPE table prefetch, TMA stores, pipelined item geometry, unmasked fast path):
# correctness first, then timing / ncu / phases; GEMM rasterisation group 8 vs 16 (traffic + time).
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or fused" > gpurun_out/r2u_kern.log 2>&1; echo "kernel tests rc=$?"; tail -3 gpurun_out/r2u_kern.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_prefix.py tests/test_gpu_whitebox.py tests/test_gpu_opt.py -q -x > gpurun_out/r2u_par.log 2>&1; echo "parity rc=$?"; tail -3 gpurun_out/r2u_par.log
for m in 14 46; do timeout 120 python tools/attn_time.py $m 512x16 32 32 10; timeout 120 python tools/attn_time.py $m 2048x16 40 40 5; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 2 -c 2 -o gpurun_out/r2u_ws_cfg1 python tools/attn_time.py 14 512x16 32 32 1 > gpurun_out/r2u_ncu1.log 2>&1; echo "ncu ws rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd -s 2 -c 2 --csv python tools/attn_time.py 14 2048x16 40 40 1 > gpurun_out/r2u_cfg3_times.csv 2>&1; echo "ncu cfg3 rc=$?"
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r2u_bench_cfg1.json 2> gpurun_out/r2u_bench_cfg1.err; echo "bench rc=$?"; head -c 400 gpurun_out/r2u_bench_cfg1.json; echo
MENOS_GEMM_GROUP_M=8 timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r2u_bench_cfg1_g8.json 2> gpurun_out/r2u_bench_cfg1_g8.err; echo "bench g8 rc=$?"
MENOS_GEMM_GROUP_M=8 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:gemm_tc_kernel -s 24 -c 8 --csv python bench.py --layers 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2u_gemm_g8.csv 2> gpurun_out/r2u_gemm_g8.err; echo "gemm g8 rc=$?"
MENOS_GEMM_GROUP_M=4 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:gemm_tc_kernel -s 24 -c 8 --csv python bench.py --layers 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2u_gemm_g4.csv 2> gpurun_out/r2u_gemm_g4.err; echo "gemm g4 rc=$?"
MENOS_NVCC_DEFS=-DMENOS_BWS_PROF timeout 600 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2u_build_prof.log 2>&1; echo "prof build rc=$?"
P=paper_conf_middleware_hul24_b200
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -I$P/csrc $P/_lib/*.o -lcuda -ldl -o /tmp/phases >> gpurun_out/r2u_build_prof.log 2>&1 && timeout 120 /tmp/phases > gpurun_out/r2u_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2u_phases.txt
