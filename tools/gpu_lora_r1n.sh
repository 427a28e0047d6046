# LoRA rows kernel: 64- vs 32-token blocks (isolated timing at cfg1 shapes), then the LoRA kernel tests + parity.
set -x
for bm in 64 32; do
  MENOS_NVCC_DEFS="-DMENOS_LORA_ROWS_BM=$bm" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $bm"
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude tools/lora_bench.cu paper_conf_middleware_hul24_b200/_lib/*.o -lcuda -o /tmp/lora_bench_$bm && echo "bm=$bm" >> gpurun_out/lora_r1n.txt && timeout 120 /tmp/lora_bench_$bm >> gpurun_out/lora_r1n.txt 2>&1
done
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_cuts.py -x -q > gpurun_out/pytest_r1n.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r1n.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_cfg1_r1n.json 2> gpurun_out/bench_cfg1_r1n.err; echo "bench rc=$?"
cat gpurun_out/lora_r1n.txt
echo done
