#!/usr/bin/env bash
# KC cold slots per thread 2/3/4 (prefix 132/120/107 KB) with the key hint: C2 + dense C5 rows
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam16.0_rho0.9,lam16.0_rho0.7,lam64.0_rho0.7,lam2.0_rho0.0
for rep in 1 2; do
timeout 1500 python scripts/variants.py run > gpurun_out/r02b7_kc_coldslots_rep$rep.log 2>&1
done
echo done
