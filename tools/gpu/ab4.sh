python -m pytest tests -m gpu -x -q -k "csr5 or coo" 2>&1 | tail -2
echo "== default"; python tools/exp.py rmat24 coo csr5 merge --reps 50
echo "== nosmap"; SPMV_CSR5_SMAP=0 python tools/exp.py rmat24 csr5 --reps 50
for c in 0 12 25 50 100; do
 echo "== carveout $c"; SPMV_CARVEOUT=$c python tools/exp.py rmat24 coo csr5 merge --reps 50
 echo "== carveout $c nosmap"; SPMV_CSR5_SMAP=0 SPMV_CARVEOUT=$c python tools/exp.py rmat24 csr5 --reps 50
done
echo "== lap carveout 0"; SPMV_CARVEOUT=0 python tools/exp.py lap4096 coo csr5 merge --reps 100
echo "== lap nosmap carveout 0"; SPMV_CSR5_SMAP=0 SPMV_CARVEOUT=0 python tools/exp.py lap4096 csr5 --reps 100
echo "== lap default"; python tools/exp.py lap4096 coo csr5 merge --reps 100
