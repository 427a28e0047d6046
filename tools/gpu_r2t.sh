# Attention-backward investigation: ncu full-set of the two-kernel (mode 14) and one-pass (mode 46) backward at the
# cfg1 (16 x 512, 32 heads) and cfg3 (16 x 2048, 40 heads) shapes; racecheck of every non-GEMM kernel after the
# epilogue barrier fix; per-phase clocks of the dK/dV kernel (-DMENOS_BWS_PROF build, last: it replaces the library).
for m in 14 46; do timeout 120 python tools/attn_time.py $m 512x16 32 32 10; timeout 120 python tools/attn_time.py $m 2048x16 40 40 5; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 2 -c 2 -o gpurun_out/r2t_ws_cfg1 python tools/attn_time.py 14 512x16 32 32 1 > gpurun_out/r2t_ncu1.log 2>&1; echo "ncu ws rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 1 -c 1 -o gpurun_out/r2t_fused_cfg1 python tools/attn_time.py 46 512x16 32 32 1 > gpurun_out/r2t_ncu2.log 2>&1; echo "ncu fused rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 2 -c 2 -o gpurun_out/r2t_ws_cfg3 python tools/attn_time.py 14 2048x16 40 40 1 > gpurun_out/r2t_ncu3.log 2>&1; echo "ncu ws cfg3 rc=$?"
MENOS_SANITIZE_MODES=14,46 timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 30 --kernel-name-exclude kns=gemm_tc_kernel python tools/sanitize_step.py > gpurun_out/r2t_racecheck_nogemm.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/r2t_racecheck_nogemm.log
MENOS_NVCC_DEFS=-DMENOS_BWS_PROF timeout 600 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2t_build_prof.log 2>&1; echo "prof build rc=$?"
P=paper_conf_middleware_hul24_b200
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -I$P/csrc $P/_lib/*.o -lcuda -ldl -o /tmp/phases >> gpurun_out/r2t_build_prof.log 2>&1 && timeout 120 /tmp/phases > gpurun_out/r2t_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2t_phases.txt
