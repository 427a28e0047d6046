timeout 1700 python -m pytest tests -m gpu -q -rf --durations=8 > gpurun_out/r2r_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -14 gpurun_out/r2r_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2r_smoke.log 2>&1; echo "smoke rc=$?"; tail -c 200 gpurun_out/r2r_smoke.log
MENOS_SANITIZE_MODES=14,46 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_step.py > gpurun_out/r2r_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -6 gpurun_out/r2r_memcheck.log
MENOS_SANITIZE_MODES=14,46 timeout 1200 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_step.py > gpurun_out/r2r_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -6 gpurun_out/r2r_racecheck.log
MENOS_SANITIZE_MODES=14,46 timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/sanitize_step.py > gpurun_out/r2r_synccheck.log 2>&1; echo "synccheck rc=$?"; tail -6 gpurun_out/r2r_synccheck.log
