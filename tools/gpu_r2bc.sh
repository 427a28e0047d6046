# LoRA dU+dB kernel v2 (rank <= 8: one n8 tile; hoisted addressing) and deeper shrink ring: parity tests, LoRA ncu at
# cfg1 / cfg3 (one layer), cfg1 bench; then the attention-backward phase clocks (-DMENOS_BWS_PROF build, last).
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_fullsize.py tests/test_gpu_opt.py tests/test_gpu_kernels.py -x -q -k "not attention" > gpurun_out/r2bc_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2bc_pytest.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:lora --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bc_lora_cfg1.csv 2> gpurun_out/r2bc_lora_cfg1.err; echo "lora ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:lora --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bc_lora_cfg3.csv 2> gpurun_out/r2bc_lora_cfg3.err; echo "lora ncu cfg3 rc=$?"
timeout 900 python bench.py --steps 10 --no-cpu-baseline > gpurun_out/r2bc_bench_cfg1.json 2> gpurun_out/r2bc_bench_cfg1.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2bc_bench_cfg1.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
MENOS_NVCC_DEFS=-DMENOS_BWS_PROF timeout 900 python -m paper_conf_middleware_hul24_b200.build -f > gpurun_out/r2bc_profbuild.log 2>&1; echo "prof build rc=$?"
L=paper_conf_middleware_hul24_b200/_lib
nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -Ipaper_conf_middleware_hul24_b200/csrc -Iinclude $L/*.o -lcuda -ldl -o /tmp/abp > gpurun_out/r2bc_abp_build.log 2>&1; echo "tool rc=$?"
timeout 300 /tmp/abp > gpurun_out/r2bc_attn_phases.txt 2>&1; echo "phases rc=$?"; cat gpurun_out/r2bc_attn_phases.txt
