timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" > gpurun_out/r2k_attn.log 2>&1; echo "attn rc=$?"; tail -3 gpurun_out/r2k_attn.log
timeout 600 python -m pytest tests/test_gpu_prefix.py -q -x > gpurun_out/r2k_prefix.log 2>&1; echo "prefix rc=$?"; tail -30 gpurun_out/r2k_prefix.log
for v in 46 14; do MENOS_ATTN_TC=$v timeout 300 python bench.py --layers 4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2k_b4_$v.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r2k_b4_$v.json').read().strip().splitlines()[-1]); k=d['kernels']['attn_bwd']; print('mode $v', round(d['ms_per_step'],2), k)"; done
MENOS_ATTN_TC=46 timeout 300 python bench.py --workload cfg3_13b_x16 --layers 2 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/r2k_c3_46.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/r2k_c3_46.json').read().strip().splitlines()[-1]); k=d['kernels']['attn_bwd']; print('cfg3 46', round(d['ms_per_step'],2), k)"
MENOS_NVCC_DEFS=-DMENOS_ABF_PROF timeout 600 python -c 'from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)' > gpurun_out/r2k_build.log 2>&1; echo "build rc=$?"
timeout 300 python tools/abf_prof.py 512x16 32 32 > gpurun_out/r2k_prof_cfg1.json 2>&1; cat gpurun_out/r2k_prof_cfg1.json
