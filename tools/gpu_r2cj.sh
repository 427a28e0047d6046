# ncu --set full of the dS-stored attention backward kernels (dK/dV + dQ-from-dS) at cfg1's shape, application
# replay (kernel replay of tcgen05 kernels ended in LaunchFailed before, r2bj / r2bk).
timeout 1500 ncu --set full --replay-mode application --clock-control none --import-source on -k regex:"attn_bwd_d" -s 2 -c 2 -o gpurun_out/r2cj_attn_bwd python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2cj_ncu.log 2>&1; echo "ncu rc=$?"; tail -5 gpurun_out/r2cj_ncu.log
ls -la gpurun_out/r2cj_attn_bwd.ncu-rep && ncu -i gpurun_out/r2cj_attn_bwd.ncu-rep --page raw --csv > gpurun_out/r2cj_raw.csv 2>/dev/null; echo "raw rc=$?"
ncu -i gpurun_out/r2cj_attn_bwd.ncu-rep --page details --csv > gpurun_out/r2cj_details.csv 2>/dev/null; echo "details rc=$?"
