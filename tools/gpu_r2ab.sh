# cfg3 bench re-run (r2aa's device-timed step had 0.46 s of gaps); ncu full-set of the LoRA rows / tokred kernels at
# cfg3 (one layer: the gate|up dU and the qkv shrink are the slowest launches).
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2ab_bench_cfg3.json 2> gpurun_out/r2ab_bench_cfg3.err; echo "cfg3 rc=$?"
timeout 600 python bench.py --workload cfg3_13b_x16 --steps 3 --no-cpu-baseline > gpurun_out/r2ab_bench_cfg3b.json 2> gpurun_out/r2ab_bench_cfg3b.err; echo "cfg3b rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lora -s 10 -c 10 -o gpurun_out/r2ab_lora python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2ab_ncu.log 2>&1; echo "ncu rc=$?"
