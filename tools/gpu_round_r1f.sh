# One GPU call: full GPU suite, smoke, default bench line, OPT-1.3B (NEXT-4) line, cfg2 line, cfg4 TP-8 rank-0
# shard compute timing (not a bench value).
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r1f.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu_r1f.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r1f.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1f.json 2> gpurun_out/bench_cfg1_r1f.err; echo "bench rc=$?"
timeout 900 python bench.py --workload opt13_x16_paper --steps 5 --no-cpu-baseline > gpurun_out/bench_opt_r1f.json 2> gpurun_out/bench_opt_r1f.err; echo "opt rc=$?"
timeout 900 python bench.py --workload cfg2_7b_x32_ragged --steps 3 --no-cpu-baseline > gpurun_out/bench_cfg2_r1f.json 2> gpurun_out/bench_cfg2_r1f.err; echo "cfg2 rc=$?"
timeout 900 python bench.py --workload cfg4_70b_tp8_x16 --tp-shard-only 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg4_shard_r1f.json 2> gpurun_out/bench_cfg4_shard_r1f.err; echo "cfg4 rc=$?"
echo done
