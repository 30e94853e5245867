#!/bin/bash
# configs[3] fp64 sweep + the every-10th stability rerun on the current kernels
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/sw
rm -f gpurun_out/sw/*.jsonl
timeout 1800 python -m paper_conf_ipps_nisassvs18_b200.harness --count 2000 --dtype f64 --out gpurun_out/sw/sweep2000_f64.jsonl > gpurun_out/sw/sweep_f64.log 2>&1
echo "f64 $?"; tail -1 gpurun_out/sw/sweep_f64.log
timeout 900 python -m paper_conf_ipps_nisassvs18_b200.harness --count 2000 --stride 10 --dtype f64 --out gpurun_out/sw/stability_f64_run2.jsonl > gpurun_out/sw/stab.log 2>&1
echo "stab $?"; tail -1 gpurun_out/sw/stab.log
python tools/label_stability.py gpurun_out/sw/sweep2000_f64.jsonl gpurun_out/sw/stability_f64_run2.jsonl --out gpurun_out/sw/label_stability_f64.json
wc -l gpurun_out/sw/*.jsonl
