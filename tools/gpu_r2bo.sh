# dQ-from-dS items: query-block order rotated per (sequence, head) group (round-robin load balance).  Attention /
# parity tests, ncu times at cfg1 / cfg3, cfg1 bench.
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -x -q -k "attention or parity or chunk" > gpurun_out/r2bo_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r2bo_tests.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bo_ncu_cfg1.csv 2> /dev/null; echo "ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bo_ncu_cfg3.csv 2> /dev/null; echo "ncu cfg3 rc=$?"
timeout 900 python bench.py --steps 10 --no-cpu-baseline > gpurun_out/r2bo_bench_cfg1.json 2> gpurun_out/r2bo_bench_cfg1.err; echo "bench rc=$?"; tail -2 gpurun_out/r2bo_bench_cfg1.err
python -c "import json;d=json.load(open('gpurun_out/r2bo_bench_cfg1.json'));print(round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks'])"
