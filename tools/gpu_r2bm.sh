# dK/dV kernel: lse / D brought by the TMA warp with each Q / dO stage (bulk copies) instead of per-thread cp.async
# one group block ahead: attention + parity tests, ncu times (same method as r2bf), cfg1 bench, phase clocks.
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_prefix.py tests/test_gpu_opt.py tests/test_gpu_cuts.py -x -q > gpurun_out/r2bm_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r2bm_tests.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bm_ncu_cfg1.csv 2> /dev/null; echo "ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bm_ncu_cfg3.csv 2> /dev/null; echo "ncu cfg3 rc=$?"
timeout 900 python bench.py --steps 10 --no-cpu-baseline > gpurun_out/r2bm_bench_cfg1.json 2> gpurun_out/r2bm_bench_cfg1.err; echo "bench rc=$?"; tail -2 gpurun_out/r2bm_bench_cfg1.err
python -c "import json;d=json.load(open('gpurun_out/r2bm_bench_cfg1.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
MENOS_NVCC_DEFS=-DMENOS_BWS_PROF timeout 900 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2bm_profbuild.log 2>&1; echo "prof build rc=$?"
L=paper_conf_middleware_hul24_b200/_lib
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -Ipaper_conf_middleware_hul24_b200/csrc -Iinclude $L/*.o -lcuda -ldl -o /tmp/abp > gpurun_out/r2bm_abp_build.log 2>&1; echo "tool rc=$?"
timeout 300 /tmp/abp ds > gpurun_out/r2bm_attn_phases_ds.txt 2>&1; echo "phases ds rc=$?"; cat gpurun_out/r2bm_attn_phases_ds.txt
