# Final measurement call of the round on the committed code (after the 256-column dU+dB slabs): full GPU suite +
# smoke, default bench (driver K/W), the reference arm, cfg2 / cfg3 / OPT lines, ncu launch list of one cfg1 step,
# metric-only per-kernel DRAM bytes of one layer (cfg1).
timeout 1500 python -m pytest tests -m gpu -x -q -rf --durations=5 > gpurun_out/r2cg_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2cg_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2cg_smoke.log 2>&1; echo "smoke rc=$?"; tail -c 300 gpurun_out/r2cg_smoke.log; echo
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2cg_bench_cfg1.json 2> gpurun_out/r2cg_bench_cfg1.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r2cg_bench_ref.json 2> gpurun_out/r2cg_bench_ref.err; echo "ref rc=$?"
timeout 600 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/r2cg_bench_cfg2.json 2> gpurun_out/r2cg_bench_cfg2.err; echo "cfg2 rc=$?"
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2cg_bench_cfg3.json 2> gpurun_out/r2cg_bench_cfg3.err; echo "cfg3 rc=$?"
timeout 600 python bench.py --workload opt13_x16_paper --steps 3 --no-cpu-baseline > gpurun_out/r2cg_bench_opt13.json 2> gpurun_out/r2cg_bench_opt13.err; echo "opt rc=$?"
for f in cfg1 cfg2 cfg3 opt13; do python -c "import json;d=json.load(open('gpurun_out/r2cg_bench_$f.json'));print('$f', round(d['value']), d.get('e2e',{}) and round(d['e2e']['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks']['sm_mhz'], round(d['roofline']['frac'],3))"; done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2cg_launches.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2cg_ncu_launch.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active --clock-control none --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2cg_layer_kernels.csv 2> gpurun_out/r2cg_layer_kernels.err; echo "layer kernels rc=$?"
