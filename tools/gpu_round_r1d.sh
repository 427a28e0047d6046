# One GPU call (round 1, session d): client sweep, cfg2 / cfg3 bench lines, ncu launch list of one cfg1 step, ncu
# full-set of the GEMM and attention kernels.  Outputs land in gpurun_out/ (summaries copied to profiles/).
set -x
timeout 600 python tools/sweep_clients.py --ns 1,4 --layers 2 --steps 1 --warmup 1 > gpurun_out/sweep_smoke.jsonl 2> gpurun_out/sweep_smoke.err
timeout 1200 python tools/sweep_clients.py > gpurun_out/sweep_r1d.jsonl 2> gpurun_out/sweep_r1d.err
timeout 900 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/bench_cfg2_r1d.json 2> gpurun_out/bench_cfg2_r1d.err
timeout 900 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/bench_cfg3_r1d.json 2> gpurun_out/bench_cfg3_r1d.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1d.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_r1d.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_.*_ws|rmsnorm|lora" -s 40 -c 16 -o gpurun_out/prof_r1d python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_r1d.log 2>&1
echo done
