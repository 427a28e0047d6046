# Fused LoRA dU+dB (one pass over dY per target) and one-pass dA per client-group: full GPU suite, cfg1 bench,
# LoRA kernel launch times + DRAM bytes for one cfg1 layer and one cfg3 layer.
timeout 1500 python -m pytest tests -m gpu -x -q -rf --durations=5 > gpurun_out/r2bb_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/r2bb_pytest_gpu.log
timeout 900 python bench.py --steps 10 --no-cpu-baseline > gpurun_out/r2bb_bench_cfg1.json 2> gpurun_out/r2bb_bench_cfg1.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2bb_bench_cfg1.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:lora --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bb_lora_cfg1.csv 2> gpurun_out/r2bb_lora_cfg1.err; echo "lora ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:lora --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bb_lora_cfg3.csv 2> gpurun_out/r2bb_lora_cfg3.err; echo "lora ncu cfg3 rc=$?"
