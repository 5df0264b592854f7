#!/usr/bin/env bash
# KL per-launch row policy (label tests + bench); KC RAW-slab index loads evict_first A/B (RAW C5 rows, C2)
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_labels.py tests/test_gpu_parity.py -q -x -k "label or raw_slab or cosmo_presets or localized" > gpurun_out/r02b6_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02b6_pytest.log
timeout 600 python scripts/label_bench.py > gpurun_out/r02b6_label_bench.json 2> gpurun_out/r02b6_label_bench.err
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam64.0_rho0.0,lam2.0_rho0.7
for rep in 1 2; do
timeout 1200 python scripts/variants.py run > gpurun_out/r02b6_kc_raw_ef_rep$rep.log 2>&1
done
echo done
