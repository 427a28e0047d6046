# Full GPU suite + smoke after the attention-backward rework; cfg1 / cfg3 bench lines; LoRA side kernels at cfg3
# (per-launch time and DRAM bytes, one layer).
timeout 1700 python -m pytest tests -m gpu -q -rf --durations=5 > gpurun_out/r2aa_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/r2aa_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2aa_smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > gpurun_out/r2aa_bench_cfg1.json 2> gpurun_out/r2aa_bench_cfg1.err; echo "bench rc=$?"; head -c 300 gpurun_out/r2aa_bench_cfg1.json; echo
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2aa_bench_cfg3.json 2> gpurun_out/r2aa_bench_cfg3.err; echo "cfg3 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:lora --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2aa_lora_cfg3.csv 2> gpurun_out/r2aa_lora_cfg3.err; echo "lora ncu rc=$?"
