#!/usr/bin/env bash
# KC diagnostic (timing only, wrong output): cold keys as one predicated global 8-B load
# (no cold slots, no conversion) vs the kept kernel vs all-hot
set -u
mkdir -p gpurun_out
VARIANTS_JSON='{"base": [], "diag_ldg": ["SPP_KC_DIAG_LDG=1"], "diag_nocold": ["SPP_KC_DIAG_NOCOLD=1"]}' VARIANT_DEEPCAM=0 \
  VARIANT_SWEEP="lam2.0_rho0.7,lam2.0_rho0.0,lam16.0_rho0.9,lam16.0_rho0.0,lam64.0_rho0.7" \
  timeout 2400 python scripts/variants.py run > gpurun_out/r02s_kc_diag_ldg.log 2>&1
echo done
