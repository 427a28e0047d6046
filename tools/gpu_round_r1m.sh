# One GPU call: full GPU suite on the committed state, default bench line, launch list of one cfg1 step, ncu
# full set of the GEMMs (incl. the SwiGLU-bwd and D-row-sum epilogues) + persistent attention kernels + RMSNorm/LoRA.
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r1m.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r1m.log
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1m.json 2> gpurun_out/bench_cfg1_r1m.err; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1m.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_r1m.log 2>&1; echo "ncu launches rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_.*_ws|rmsnorm|lora_" -s 60 -c 20 -o gpurun_out/prof_r1m python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_r1m.log 2>&1; echo "ncu full rc=$?"
tail -3 gpurun_out/ncu_full_r1m.log
echo done
