#!/usr/bin/env bash
# same-box A/B: RAW-slab loop (new vs round-1) and key-tile evict_first on C2 and the dense C5 rows
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam64.0_rho0.0,lam16.0_rho0.9,lam2.0_rho0.0
for rep in 1 2; do
timeout 1200 python scripts/variants.py run > gpurun_out/r02a5_kc_raw_keyef_rep$rep.log 2>&1
done
echo done
