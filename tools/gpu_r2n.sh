timeout 300 python tools/dbg_prefix_nograd.py > gpurun_out/r2n_dbg.log 2>&1; echo "dbg rc=$?"; cat gpurun_out/r2n_dbg.log | tail -6
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" > gpurun_out/r2n_attn.log 2>&1; echo "attn rc=$?"; tail -5 gpurun_out/r2n_attn.log
timeout 900 python -m pytest tests/test_gpu_opt.py tests/test_gpu_prefix.py tests/test_gpu_tp.py -q > gpurun_out/r2n_t.log 2>&1; echo "t rc=$?"; grep -E "^E   .{0,300}|passed|failed" gpurun_out/r2n_t.log | cut -c1-300 | tail -12
timeout 300 python bench.py --workload opt13_x16_paper --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2n_opt.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r2n_opt.json').read().strip().splitlines()[-1]); print('opt', d['value'], d['ms_per_step']); [print(k, v) for k, v in d['kernels'].items()]"
