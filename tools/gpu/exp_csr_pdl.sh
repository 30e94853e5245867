python tools/exp.py rmat24 csr csr:csr_chunk=2048 csr:csr_chunk=256 > gpurun_out/exp_csr3.log 2>&1
SPMV_CSR_PDL=0 python tools/exp.py rmat24 csr >> gpurun_out/exp_csr3.log 2>&1
SPMV_CSR_CHUNK_CTAS=1 python tools/exp.py rmat24 csr >> gpurun_out/exp_csr3.log 2>&1
SPMV_CSR_CHUNK_CTAS=4 python tools/exp.py rmat24 csr >> gpurun_out/exp_csr3.log 2>&1
python tools/exp.py rmat24 csr --dtype f32 >> gpurun_out/exp_csr3.log 2>&1
python -m pytest tests -m gpu -x -q 2>&1 | tail -5 >> gpurun_out/exp_csr3.log
