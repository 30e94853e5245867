python -m pytest tests -m gpu -x -q -k "csr5" 2>&1 | tail -2
for i in 1 2; do
echo "== smap"; python tools/exp.py rmat24 csr5 merge --reps 50
echo "== nosmap"; SPMV_CSR5_SMAP=0 python tools/exp.py rmat24 csr5 --reps 50
done
python tools/exp.py rmat24 csr5 --dtype f32 --reps 50
SPMV_CSR5_SMAP=0 python tools/exp.py rmat24 csr5 --dtype f32 --reps 50
python tools/exp.py lap4096 csr5 --reps 100
SPMV_CSR5_SMAP=0 python tools/exp.py lap4096 csr5 --reps 100
