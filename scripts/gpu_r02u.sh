#!/usr/bin/env bash
# KC cold rows loaded directly in the expansion (no lookahead slots): C2 + dense sweep A/B
# (first run, r02u: separate raw-row array -> spills; second run, r02u2: rows loaded into the entries in place)
set -u
mkdir -p gpurun_out
VARIANTS_JSON='{"base": [], "direct": ["SPP_KC_COLD_DIRECT=1"], "direct_la0": ["SPP_KC_COLD_DIRECT=1", "SPP_KC_LA=0"]}' VARIANT_DEEPCAM=0 \
  VARIANT_SWEEP="lam2.0_rho0.7,lam2.0_rho0.0,lam16.0_rho0.9,lam16.0_rho0.0,lam64.0_rho0.7" \
  timeout 2400 python scripts/variants.py run > gpurun_out/r02u2_kc_cold_direct.log 2>&1
echo done
