# Three-deep work-item geometry pipeline in the attention backward: kernel tests, ncu times (cfg1 / cfg3, same
# method as r2bf), and compute-sanitizer memcheck / racecheck / synccheck over the default path (mode 78) and the
# recompute path (mode 14) including the new tcgen05 LoRA kernels.
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "attention" > gpurun_out/r2bl_attn.log 2>&1; echo "attn tests rc=$?"; tail -2 gpurun_out/r2bl_attn.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2bl_ncu_cfg1.csv 2> /dev/null; echo "ncu cfg1 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --workload cfg3_13b_x16 --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --arena-gb 60 > gpurun_out/r2bl_ncu_cfg3.csv 2> /dev/null; echo "ncu cfg3 rc=$?"
MENOS_SANITIZE_MODES=78,14 timeout 1200 compute-sanitizer --tool memcheck python tools/sanitize_step.py > gpurun_out/r2bl_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/r2bl_memcheck.log
MENOS_SANITIZE_MODES=78 timeout 1200 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 30 --kernel-name-exclude kns=gemm_tc_kernel python tools/sanitize_step.py > gpurun_out/r2bl_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/r2bl_racecheck.log
MENOS_SANITIZE_MODES=78 timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize_step.py > gpurun_out/r2bl_synccheck.log 2>&1; echo "synccheck rc=$?"; tail -3 gpurun_out/r2bl_synccheck.log
