# One GPU call: full GPU suite, smoke, default bench line, cfg3 bench, launch list, ncu full-set of the GEMM and
# attention-backward kernels (arena capped so the replay's memory save/restore stays small).
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r1e.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_r1e.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r1e.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1e.json 2> gpurun_out/bench_cfg1_r1e.err; echo "bench rc=$?"
timeout 900 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/bench_cfg3_r1e.json 2> gpurun_out/bench_cfg3_r1e.err; echo "cfg3 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1e.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/ncu_launch_r1e.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_bwd_.*_ws|attn_fwd_ws|lora_rows|layernorm|rmsnorm_bwd" -s 40 -c 14 -o gpurun_out/prof_r1e python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --arena-gb 40 > gpurun_out/ncu_full_r1e.log 2>&1
echo done
