# LayerNorm (OPT): per-row named barriers instead of CTA-wide syncs, mean(gh) and mean(gh xh) in one exchange.
timeout 900 python -m pytest tests/test_gpu_opt.py tests/test_gpu_kernels.py -x -q -k "opt or layernorm or OPT" > gpurun_out/r2cc_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/r2cc_tests.log
timeout 600 python bench.py --workload opt13_x16_paper --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2cc_bench_opt13.json 2> gpurun_out/r2cc_bench_opt13.err; echo "opt rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2cc_bench_opt13.json'));print('opt', round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['kernels']['rmsnorm'].get('frac_hbm'), d['clocks']['sm_mhz'])"
