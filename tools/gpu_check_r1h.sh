# One GPU call (session r1h, after container restore): full GPU suite, smoke, default bench line.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_r1h.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r1h.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r1h.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke_r1h.log
timeout 900 python bench.py > gpurun_out/bench_cfg1_r1h.json 2> gpurun_out/bench_cfg1_r1h.err; echo "bench rc=$?"
echo done
