#!/usr/bin/env bash
# KC: f(U) staged in shared memory as 16-bit output values (fu16) vs fp32 (fu32): C2 + dense C5 rows, 2 reps
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam64.0_rho0.0,lam16.0_rho0.9,lam2.0_rho0.0,lam2.0_rho0.7
for rep in 1 2; do
timeout 1200 python scripts/variants.py run > gpurun_out/r02a9_kc_fu16_rep$rep.log 2>&1
done
echo done
