#!/usr/bin/env bash
# KC shape variants with the key evict_first hint: consumer threads 768/640/512 (more registers,
# longer hot prefix) and key-ring depth 4/6 (prefix 144/120 KB); C2 + dense C5 rows, 2 reps
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam16.0_rho0.9,lam2.0_rho0.0,lam2.0_rho0.7,lam64.0_rho0.7
for rep in 1 2; do
timeout 1500 python scripts/variants.py run > gpurun_out/r02b4_kc_shape_rep$rep.log 2>&1
done
echo done
