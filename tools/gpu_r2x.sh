# lse / D by cp.async two blocks ahead into a 3-slot ring (dK/dV kernel); 8 vs 16 softmax-gradient warps.
P=paper_conf_middleware_hul24_b200
times() {
  for shp in "512x16 32 32" "2048x16 40 40" "512x16 64 64 5 64"; do
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:attn_bwd -s 2 -c 2 --csv python tools/attn_time.py 14 $shp 1 2>/dev/null | grep gpu__time | awk -F'","' -v s="$shp" '{print s, substr($5,1,40), $NF}'
  done
}
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or fused" > gpurun_out/r2x_kern.log 2>&1; echo "kernel tests rc=$?"; tail -2 gpurun_out/r2x_kern.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_prefix.py -q -x > gpurun_out/r2x_par.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/r2x_par.log
echo "== EW 8"; times
MENOS_NVCC_DEFS="-DMENOS_BWS_EW=16" timeout 600 python -m $P.build -f > gpurun_out/r2x_build16.log 2>&1; echo "build16 rc=$?"
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention or fused" > gpurun_out/r2x_kern16.log 2>&1; echo "kernel tests (EW 16) rc=$?"; tail -2 gpurun_out/r2x_kern16.log
echo "== EW 16"; times
MENOS_NVCC_DEFS="-DMENOS_BWS_PROF" timeout 600 python -m $P.build -f > gpurun_out/r2x_build_prof.log 2>&1
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -I$P/csrc $P/_lib/*.o -lcuda -ldl -o /tmp/phases >> gpurun_out/r2x_build_prof.log 2>&1 && timeout 120 /tmp/phases > gpurun_out/r2x_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2x_phases.txt
