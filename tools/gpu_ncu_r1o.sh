# ncu captures split per kernel family (the combined --set full capture fails with LaunchFailed on this build):
# which family fails under full-set instrumentation, plus an un-instrumented section set over all hot kernels.
set -x
B="python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc_kernel -s 40 -c 4 -o gpurun_out/prof_r1o_gemm $B > gpurun_out/ncu_r1o_gemm.log 2>&1; echo "gemm rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_fwd_ws -s 6 -c 1 -o gpurun_out/prof_r1o_afwd $B > gpurun_out/ncu_r1o_afwd.log 2>&1; echo "afwd rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd -s 12 -c 2 -o gpurun_out/prof_r1o_abwd $B > gpurun_out/ncu_r1o_abwd.log 2>&1; echo "abwd rc=$?"
timeout 600 ncu --set full --clock-control none -k regex:"rmsnorm|lora_" -s 40 -c 8 -o gpurun_out/prof_r1o_misc $B > gpurun_out/ncu_r1o_misc.log 2>&1; echo "misc rc=$?"
timeout 900 ncu --section SpeedOfLight --section MemoryWorkloadAnalysis --section LaunchStats --section Occupancy --metrics dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:"gemm_tc_kernel|attn_fwd_ws|attn_bwd_.*_ws|rmsnorm|lora_|adamw" -s 60 -c 24 -o gpurun_out/prof_r1o_sol $B > gpurun_out/ncu_r1o_sol.log 2>&1; echo "sol rc=$?"
for f in gemm afwd abwd misc sol; do grep -c "==PROF== Profiling" gpurun_out/ncu_r1o_$f.log; grep "ERROR" gpurun_out/ncu_r1o_$f.log | head -2; done
echo done
