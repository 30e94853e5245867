python -m pytest tests -m gpu -x -q -k "merge" 2>&1 | tail -1
SPMV_CSR_FLAT=12 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "csr and not csr5 and not scalar" 2>&1 | tail -1
SPMV_CSR_FLAT=8 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "csr and not csr5 and not scalar" 2>&1 | tail -1
for dt in f64 f32; do
for i in 1 2; do
echo "== base $dt"; SPMV_LIB_PATH=tools/ab/libspmv_base.so python tools/exp.py lap4096 merge csr --dtype $dt --reps 200
echo "== new $dt"; python tools/exp.py lap4096 merge --dtype $dt --reps 200
for j in 8 10 12; do echo "== flat $j $dt"; SPMV_CSR_FLAT=$j python tools/exp.py lap4096 csr --dtype $dt --reps 200; done
done; done
echo "== rmat base"; SPMV_LIB_PATH=tools/ab/libspmv_base.so python tools/exp.py rmat24 merge --reps 50
echo "== rmat new"; python tools/exp.py rmat24 merge --reps 50
