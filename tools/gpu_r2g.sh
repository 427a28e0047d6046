MENOS_NVCC_DEFS=-DMENOS_ABF_PROF timeout 600 python -c 'from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)' > gpurun_out/r2g_build.log 2>&1; echo "build rc=$?"
for m in 0 1 4; do MENOS_ABF_DBG=$m timeout 300 python tools/abf_prof.py 512x16 32 32 > gpurun_out/r2g_prof_cfg1_$m.json 2>&1; cat gpurun_out/r2g_prof_cfg1_$m.json; done
