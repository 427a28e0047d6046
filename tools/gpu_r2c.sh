# fused attention backward diagnosis: variants timed in a 4-layer cfg1 step, then one ncu capture
for m in 0 1 2 3; do MENOS_ABF_DBG=$m timeout 300 python bench.py --layers 4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2c_dbg$m.json 2>/dev/null; echo "dbg $m rc=$?"; done
MENOS_ATTN_TC=14 timeout 300 python bench.py --layers 4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2c_ws.json 2>/dev/null; echo "ws rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_bwd_fused -s 2 -c 1 -o gpurun_out/r2c_abf python bench.py --layers 2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2c_ncu.log 2>&1; echo "ncu rc=$?"
timeout 600 python -m pytest tests/test_gpu_api.py tests/test_gpu_tp.py -q -x > gpurun_out/r2c_tp.log 2>&1; echo "tp rc=$?"; tail -5 gpurun_out/r2c_tp.log
free -g | head -2; nproc
