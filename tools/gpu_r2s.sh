# Round-2 measurement call: bench lines (cfg1 default, reference arm, cfg2, cfg3, OPT paper setting, TP-8 shard),
# the ncu launch list of one cfg1 step, per-GEMM DRAM traffic of one layer, an ncu full-set capture of the GEMM and
# attention kernels, and racecheck over every kernel family except the GEMM (whose only report is tcgen05.alloc).
timeout 900 python bench.py > gpurun_out/r2s_bench_cfg1.json 2> gpurun_out/r2s_bench_cfg1.err; echo "bench rc=$?"; cat gpurun_out/r2s_bench_cfg1.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r2s_bench_ref.json 2> gpurun_out/r2s_bench_ref.err; echo "ref rc=$?"
timeout 600 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/r2s_bench_cfg2.json 2> gpurun_out/r2s_bench_cfg2.err; echo "cfg2 rc=$?"
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2s_bench_cfg3.json 2> gpurun_out/r2s_bench_cfg3.err; echo "cfg3 rc=$?"
timeout 600 python bench.py --workload opt13_x16_paper --steps 3 --no-cpu-baseline > gpurun_out/r2s_bench_opt13.json 2> gpurun_out/r2s_bench_opt13.err; echo "opt rc=$?"
timeout 600 python bench.py --workload cfg4_70b_tp8_x16 --tp-shard-only 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r2s_cfg4_tp8_shard_NOT_A_BENCH_VALUE.json 2> gpurun_out/r2s_cfg4.err; echo "cfg4 rc=$?"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2s_launches.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2s_ncu_launch.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:gemm_tc_kernel -s 24 -c 8 --csv python bench.py --layers 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2s_gemm.csv 2> gpurun_out/r2s_gemm.err; echo "gemm traffic rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_.*_ws|rmsnorm|lora" -s 60 -c 24 -o gpurun_out/r2s_prof python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2s_ncu_full.log 2>&1; echo "ncu full rc=$?"
MENOS_SANITIZE_MODES=14 timeout 900 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 50 --kernel-name-exclude kns=gemm_tc_kernel python tools/sanitize_step.py > gpurun_out/r2s_racecheck_nogemm.log 2>&1; echo "racecheck rc=$?"; tail -4 gpurun_out/r2s_racecheck_nogemm.log
