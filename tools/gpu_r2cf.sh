# dU+dB kernel with 256-column slabs for the wide targets (N_t >= 8192): parity/bitwise tests, then per-kernel
# times at cfg3 (gate/up targeted) with the new default and MENOS_LORA_DUB_MT=128 (the previous kernel)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cuts.py tests/test_gpu_parity_fullsize.py -m gpu -x -q -rf > gpurun_out/r2cf_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2cf_pytest.log
for mt in 0 128; do
MENOS_LORA_DUB_MT=$mt timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"lora_d" --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2cf_ncu_cfg3_mt$mt.csv 2> /dev/null; echo "ncu cfg3 mt=$mt rc=$?"
done
for mt in 0 128; do
MENOS_LORA_DUB_MT=$mt timeout 900 python bench.py --workload cfg3_13b_x16 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --arena-gb 60 > gpurun_out/r2cf_bench_cfg3_mt$mt.json 2> gpurun_out/r2cf_bench_cfg3_mt$mt.err; echo "bench cfg3 mt=$mt rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2cf_bench_cfg3_mt$mt.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks']['sm_mhz'])"
done
