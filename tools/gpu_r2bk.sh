# ncu full-set captures of the non-GEMM kernels of a 2-layer cfg1 step (the GEMM hits LaunchFailed under full-set
# replay, r2bj), and the attention-backward phase clocks on the dS-stored path.
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"attn_fwd_ws|attn_bwd_dkdv|attn_bwd_dq_ds|rmsnorm_bwd|lora_dub_tc|lora_shrink_tc|lora_da_tc|lora_du_reduce" -c 10 -o gpurun_out/r2bk_prof python bench.py --layers 2 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bk_ncu_full.log 2>&1; echo "ncu full rc=$?"
MENOS_NVCC_DEFS=-DMENOS_BWS_PROF timeout 900 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2bk_profbuild.log 2>&1; echo "prof build rc=$?"
L=paper_conf_middleware_hul24_b200/_lib
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -Ipaper_conf_middleware_hul24_b200/csrc -Iinclude $L/*.o -lcuda -ldl -o /tmp/abp > gpurun_out/r2bk_abp_build.log 2>&1; echo "tool rc=$?"
timeout 300 /tmp/abp ds > gpurun_out/r2bk_attn_phases_ds.txt 2>&1; echo "phases ds rc=$?"; cat gpurun_out/r2bk_attn_phases_ds.txt
timeout 300 /tmp/abp > gpurun_out/r2bk_attn_phases_recompute.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2bk_attn_phases_recompute.txt
