# lse / D two blocks ahead in the dK/dV kernel, next-item row statistics after block 0 in the dQ kernel.
P=paper_conf_middleware_hul24_b200
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or fused" > gpurun_out/r2w_kern.log 2>&1; echo "kernel tests rc=$?"; tail -2 gpurun_out/r2w_kern.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_prefix.py -q -x > gpurun_out/r2w_par.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/r2w_par.log
for shp in "512x16 32 32" "2048x16 40 40" "512x16 64 64 5 64"; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd -s 2 -c 2 --csv python tools/attn_time.py 14 $shp 1 2>/dev/null | grep gpu__time | awk -F'","' -v s="$shp" '{print s, substr($5,1,40), $NF}'
done
MENOS_NVCC_DEFS="-DMENOS_BWS_PROF" timeout 600 python -m $P.build -f > gpurun_out/r2w_build_prof.log 2>&1
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -I$P/csrc $P/_lib/*.o -lcuda -ldl -o /tmp/phases >> gpurun_out/r2w_build_prof.log 2>&1 && timeout 120 /tmp/phases > gpurun_out/r2w_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2w_phases.txt
