# Forward attention phase clocks (-DMENOS_WS_PROF build; replaces the library, so last).
MENOS_NVCC_DEFS=-DMENOS_WS_PROF timeout 900 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2bz_profbuild.log 2>&1; echo "prof build rc=$?"
L=paper_conf_middleware_hul24_b200/_lib
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_fwd_phases.cu -Ipaper_conf_middleware_hul24_b200/csrc -Iinclude $L/*.o -lcuda -ldl -o /tmp/afp > gpurun_out/r2bz_afp_build.log 2>&1; echo "tool rc=$?"; tail -3 gpurun_out/r2bz_afp_build.log
timeout 300 /tmp/afp > gpurun_out/r2bz_attn_fwd_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2bz_attn_fwd_phases.txt
