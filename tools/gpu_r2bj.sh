# Round-2 session-b measurement call: full GPU suite + smoke, the default bench line (driver's K/W), the reference
# arm, cfg2 / cfg3 / OPT / cfg4-shard lines, the ncu launch list of one cfg1 step, and ncu full-set captures of the
# main kernels (2-layer cfg1 step).
timeout 1500 python -m pytest tests -m gpu -x -q -rf --durations=5 > gpurun_out/r2bj_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 gpurun_out/r2bj_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bj_smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/r2bj_smoke.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2bj_bench_cfg1.json 2> gpurun_out/r2bj_bench_cfg1.err; echo "bench rc=$?"; head -c 600 gpurun_out/r2bj_bench_cfg1.json; echo
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r2bj_bench_ref.json 2> gpurun_out/r2bj_bench_ref.err; echo "ref rc=$?"
timeout 600 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/r2bj_bench_cfg2.json 2> gpurun_out/r2bj_bench_cfg2.err; echo "cfg2 rc=$?"
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2bj_bench_cfg3.json 2> gpurun_out/r2bj_bench_cfg3.err; echo "cfg3 rc=$?"
timeout 600 python bench.py --workload opt13_x16_paper --steps 3 --no-cpu-baseline > gpurun_out/r2bj_bench_opt13.json 2> gpurun_out/r2bj_bench_opt13.err; echo "opt rc=$?"
timeout 600 python bench.py --workload cfg4_70b_tp8_x16 --tp-shard-only 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r2bj_cfg4_tp8_shard_NOT_A_BENCH_VALUE.json 2> gpurun_out/r2bj_cfg4.err; echo "cfg4 rc=$?"
for f in cfg1 cfg2 cfg3 opt13; do python -c "import json;d=json.load(open('gpurun_out/r2bj_bench_$f.json'));print('$f', round(d['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks']['sm_mhz'])"; done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bj_launches.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2bj_ncu_launch.log 2>&1; echo "launch list rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_dkdv|attn_bwd_dq_ds|rmsnorm_bwd|lora_dub_tc|lora_shrink_tc|lora_da_tc" -s 40 -c 16 -o gpurun_out/r2bj_prof python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2bj_ncu_full.log 2>&1; echo "ncu full rc=$?"
