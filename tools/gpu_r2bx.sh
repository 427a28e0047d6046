# Vectorised AdamW: AdamW / serving / prefix / parity tests, cfg3 and cfg1 bench (adamw ms per step).
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_serve.py tests/test_gpu_prefix.py tests/test_gpu_api.py -x -q > gpurun_out/r2bx_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r2bx_tests.log
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r2bx_bench_cfg3.json 2> gpurun_out/r2bx_bench_cfg3.err; echo "cfg3 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2bx_bench_cfg3.json'));print('cfg3', round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['kernels']['adamw'].get('gbs'))"
timeout 600 python bench.py --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2bx_bench_cfg1.json 2> /dev/null; echo "cfg1 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2bx_bench_cfg1.json'));print('cfg1', round(d['value']), d['kernels']['adamw'])"
