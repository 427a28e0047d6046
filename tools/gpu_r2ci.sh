# Wide-slab GPU tests (ranks within the server's max), and the host work per step (each call timed with the GPU
# idle) at cfg1 and cfg3.
timeout 600 python -m pytest tests/test_gpu_wide_slabs.py -m gpu -x -q -rf > gpurun_out/r2ci_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2ci_pytest.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2ci_cfg1.json 2> gpurun_out/r2ci_cfg1.err; echo "cfg1 rc=$?"
timeout 900 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r2ci_cfg3.json 2> gpurun_out/r2ci_cfg3.err; echo "cfg3 rc=$?"
for f in cfg1 cfg3; do python -c "import json;d=json.load(open('gpurun_out/r2ci_$f.json'));print('$f', round(d['value']), round(d['ms_per_step'],1), 'enqueue', round(d['host_enqueue_ms_per_step'],1), {k:round(v,1) for k,v in d['host_ms_per_call_gpu_idle'].items()}, d['config'].get('waves'))"; done
