# New wide-slab GPU tests (d_ff = 8200: 256-column dU+dB slabs), and the cfg3 headline-region anomaly of r2cg
# (1.78 s/step vs 1.56-1.58 in the events / e2e regions of the same run): host enqueue time per step, with and
# without the nvidia-smi clock sampler.
timeout 600 python -m pytest tests/test_gpu_wide_slabs.py -m gpu -x -q -rf > gpurun_out/r2ch_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2ch_pytest.log
for c in 1 0 1; do
MENOS_BENCH_CLOCKS=$c timeout 900 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2ch_cfg3_clk$c.json 2> gpurun_out/r2ch_cfg3_clk$c.err; echo "cfg3 clocks=$c rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2ch_cfg3_clk$c.json'));print(round(d['value']), round(d['ms_per_step'],1), round(d['e2e']['ms_per_step'],1), d['roofline']['region'][-40:], 'host', round(d['host_enqueue_ms_per_step'],1))"
done
