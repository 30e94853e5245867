python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for cfg in rmat24 lap4096; do python tools/exp.py $cfg coo csr5 merge --reps 50; done
python tools/exp.py rmat24 coo csr5 --dtype f32 --reps 50
