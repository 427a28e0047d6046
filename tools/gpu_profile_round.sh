# One GPU call: default bench line (cfg1), cfg2 bench, the ncu launch list of one cfg1 step, ncu full-set of
# the GEMM and persistent attention kernels (2-layer segment).  Outputs land in gpurun_out/ (copy summaries to
# profiles/ with tools/ncu_summary.py).
set -x
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1c.json 2> gpurun_out/bench_cfg1_r1c.err
timeout 900 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/bench_cfg2_r1c.json 2> gpurun_out/bench_cfg2_r1c.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1c.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_.*_ws" -s 40 -c 12 -o gpurun_out/prof_r1c python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
echo done
