timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" > gpurun_out/r2b_attn.log 2>&1; echo "attn rc=$?"; tail -30 gpurun_out/r2b_attn.log
timeout 900 python -m pytest tests/test_gpu_whitebox.py tests/test_gpu_parity.py tests/test_gpu_api.py tests/test_gpu_opt.py tests/test_gpu_parity_fullsize.py -q -x -k "not cfg1_full" > gpurun_out/r2b_par.log 2>&1; echo "par rc=$?"; tail -30 gpurun_out/r2b_par.log
timeout 600 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/r2b_bench.json 2> gpurun_out/r2b_bench.err; echo "bench rc=$?"; tail -3 gpurun_out/r2b_bench.err
