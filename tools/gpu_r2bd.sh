# dS-stored attention backward (dK/dV kernel stores dS^T tiles, dQ from the tiles): kernel tests (both paths, chunked),
# end-to-end parity, LoRA v3 (tokred 64-col tiles), cfg1 bench, attention kernel times under ncu.
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "attention" > gpurun_out/r2bd_attn.log 2>&1; echo "attn tests rc=$?"; tail -15 gpurun_out/r2bd_attn.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_fullsize.py tests/test_gpu_opt.py tests/test_gpu_cuts.py -x -q > gpurun_out/r2bd_parity.log 2>&1; echo "parity rc=$?"; tail -5 gpurun_out/r2bd_parity.log
timeout 900 python bench.py --steps 10 --no-cpu-baseline > gpurun_out/r2bd_bench_cfg1.json 2> gpurun_out/r2bd_bench_cfg1.err; echo "bench rc=$?"; tail -3 gpurun_out/r2bd_bench_cfg1.err
python -c "import json;d=json.load(open('gpurun_out/r2bd_bench_cfg1.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
MENOS_ATTN_TC=14 timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/r2bd_bench_cfg1_mode14.json 2> /dev/null; echo "bench14 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2bd_bench_cfg1_mode14.json'));print('mode14', round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd|lora" --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bd_ncu_cfg1.csv 2> gpurun_out/r2bd_ncu_cfg1.err; echo "ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bd_ncu_cfg3.csv 2> gpurun_out/r2bd_ncu_cfg3.err; echo "ncu cfg3 rc=$?"
