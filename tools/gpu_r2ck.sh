# dQ-from-dS: per-CTA runs of same-(sequence, query block) items so the epilogue loads the RoPE rows once per run
# (r2cj: the RoPE-table loads bound it).  Attention + parity tests, then per-kernel time (ncu metric pass) and the
# default bench.
timeout 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_cuts.py tests/test_gpu_parity_fullsize.py -m gpu -x -q -rf > gpurun_out/r2ck_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2ck_pytest.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"attn_bwd" --csv python bench.py --layers 1 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2ck_ncu_cfg1.csv 2> /dev/null; echo "ncu rc=$?"
python tools/ncu_layer_table.py gpurun_out/r2ck_ncu_cfg1.csv
timeout 900 python bench.py > gpurun_out/r2ck_bench_cfg1.json 2> gpurun_out/r2ck_bench_cfg1.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2ck_bench_cfg1.json'));print(round(d['value']), round(d['e2e']['value']), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items()}, d['clocks']['sm_mhz'], round(d['roofline']['frac'],3))"
