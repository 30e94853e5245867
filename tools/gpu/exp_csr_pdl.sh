# CSR launch-order experiments (A25 PDL): R-MAT 24 serial vs PDL, LAP4096 unchunked kernels
python tools/exp.py lap4096 csr --reps 200 > gpurun_out/exp_csr4.log 2>&1
python tools/exp.py lap4096 csr --reps 200 --dtype f32 >> gpurun_out/exp_csr4.log 2>&1
python tools/exp.py rmat24 csr >> gpurun_out/exp_csr4.log 2>&1
SPMV_CSR_PDL=0 python tools/exp.py rmat24 csr >> gpurun_out/exp_csr4.log 2>&1
python -m pytest tests -m gpu -x -q 2>&1 | tail -3 >> gpurun_out/exp_csr4.log
