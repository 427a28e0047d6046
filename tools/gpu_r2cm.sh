# Headline region preceded by one untimed step after the clock sampler's start-up pause: two default bench runs.
for i in 1 2; do
timeout 900 python bench.py > gpurun_out/r2cm_bench_cfg1_$i.json 2> gpurun_out/r2cm_bench_cfg1_$i.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/r2cm_bench_cfg1_$i.json'));print(round(d['value']), round(d['e2e']['value']), round(d['ms_per_step'],1), round(sum(v['ms_per_step'] for v in d['kernels'].values()),1), d['clocks']['sm_mhz'], round(d['roofline']['frac'],3))"
done
