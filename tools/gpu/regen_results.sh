# regenerate results/ with the current kernels: sweep (configs[3]) fp64 + fp32, R-MAT27 (configs[4]) on one GPU
python -m paper_conf_ipps_nisassvs18_b200.harness --count 2000 --dtype f64 --out gpurun_out/sweep2000_f64.jsonl > gpurun_out/sweep_f64.log 2>&1
python -m paper_conf_ipps_nisassvs18_b200.harness --count 2000 --dtype f32 --out gpurun_out/sweep2000_f32.jsonl > gpurun_out/sweep_f32.log 2>&1
python tools/rmat27_check.py --out gpurun_out/rmat27_check.json > gpurun_out/rmat27.log 2>&1
tail -n 2 gpurun_out/sweep_f64.log gpurun_out/sweep_f32.log gpurun_out/rmat27.log
