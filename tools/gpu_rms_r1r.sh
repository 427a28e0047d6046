# RMSNorm one-row-per-256-threads default (d <= 5120): kernel + parity tests, isolated timing, cfg1 and cfg3 bench.
set -x
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_r1r.log 2>&1; echo "pytest rc=$?"; tail -n 2 gpurun_out/pytest_r1r.log
for shp in "8192 4096" "8192 5120" "2048 4096"; do timeout 120 python tools/rms_time.py $shp >> gpurun_out/rms_r1r.txt 2>&1; done
cat gpurun_out/rms_r1r.txt
timeout 400 python bench.py > gpurun_out/bench_r1r_cfg1.json 2> gpurun_out/bench_r1r_cfg1.err; echo "bench rc=$?"
echo done
