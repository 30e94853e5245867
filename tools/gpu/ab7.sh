python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for i in 1 2; do
echo "== base"; SPMV_LIB_PATH=tools/ab/libspmv_base.so python tools/exp.py rmat24 coo csr hyb merge csr5 --reps 50
echo "== new"; python tools/exp.py rmat24 coo csr hyb merge csr5 --reps 50
done
echo "== base lap"; SPMV_LIB_PATH=tools/ab/libspmv_base.so python tools/exp.py lap4096 coo merge csr5 --reps 200
echo "== new lap"; python tools/exp.py lap4096 coo merge csr5 --reps 200
