timeout 1500 python -m pytest tests -m gpu -q -rf --durations=10 > gpurun_out/r2m_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -25 gpurun_out/r2m_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2m_smoke.log 2>&1; echo "smoke rc=$?"; tail -c 300 gpurun_out/r2m_smoke.log
timeout 900 python bench.py > gpurun_out/r2m_bench.json 2> gpurun_out/r2m_bench.err; echo "bench rc=$?"; tail -3 gpurun_out/r2m_bench.err
