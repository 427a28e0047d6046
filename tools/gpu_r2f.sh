timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -k "attention" > gpurun_out/r2f_attn.log 2>&1; echo "attn rc=$?"; tail -3 gpurun_out/r2f_attn.log
timeout 300 python bench.py --layers 4 --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/r2f_b4.json 2>/dev/null; echo "b4 rc=$?"
python -c "
import json; d=json.loads(open('gpurun_out/r2f_b4.json').read().strip().splitlines()[-1]); k=d['kernels']['attn_bwd']; print('attn_bwd', k)"
MENOS_NVCC_DEFS=-DMENOS_ABF_PROF timeout 600 python -c 'from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)' > gpurun_out/r2f_build.log 2>&1; echo "build rc=$?"
timeout 300 python tools/abf_prof.py 512x16 32 32 > gpurun_out/r2f_prof_cfg1.json 2>&1; cat gpurun_out/r2f_prof_cfg1.json
timeout 300 python tools/abf_prof.py 2048x8 40 40 > gpurun_out/r2f_prof_cfg3.json 2>&1; cat gpurun_out/r2f_prof_cfg3.json
