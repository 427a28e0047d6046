# GEMM epilogue variants (tuning aid): time the dX shapes per variant; then the GPU kernel tests on the default.
set -x
C=paper_conf_middleware_hul24_b200/csrc/gemm_tcgen05.cu
cp $C /tmp/gemm_keep.cu
run() {  # $1 tag, $2 source, $3 defs
  cp $2 $C
  MENOS_NVCC_DEFS="$3" python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build failed $1"
  timeout 300 python tools/gemm_epi_time.py $1 >> gpurun_out/epi_r1k.jsonl 2>> gpurun_out/epi_r1k.err
}




run new8 tools/_variants/gemm_new.cu "-DMENOS_GEMM_EPW=8"
run noload8 tools/_variants/gemm_noload.cu "-DMENOS_GEMM_EPW=8"
run nostore2_8 tools/_variants/gemm_nostore2.cu "-DMENOS_GEMM_EPW=8"
run nocompute8 tools/_variants/gemm_nocompute.cu "-DMENOS_GEMM_EPW=8"
run ldg8 tools/_variants/gemm_ldg.cu "-DMENOS_GEMM_EPW=8"
run noload4 tools/_variants/gemm_noload.cu "-DMENOS_GEMM_EPW=4"
run new8b tools/_variants/gemm_new.cu "-DMENOS_GEMM_EPW=8"
cp /tmp/gemm_keep.cu $C
python -c "from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q > gpurun_out/pytest_r1k.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_r1k.log
cat gpurun_out/epi_r1k.jsonl
echo done
