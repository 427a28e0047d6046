# Full GPU suite + smoke + default bench on the final commit of the round.
timeout 1500 python -m pytest tests -m gpu -x -q -rf > gpurun_out/r2cl_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2cl_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2cl_smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/r2cl_bench_cfg1.json 2> gpurun_out/r2cl_bench_cfg1.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2cl_bench_cfg1.json'));print(round(d['value']), round(d['e2e']['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks']['sm_mhz'], round(d['roofline']['frac'],3))"
