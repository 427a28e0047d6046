# New memory-bound test for the dS-stored backward (hd 128) + the parity file.
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r2bp_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/r2bp_tests.log
