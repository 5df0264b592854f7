#!/usr/bin/env bash
# KC: a thread's cold positions in one loop vs one divergent branch per position
set -u
mkdir -p gpurun_out
VARIANTS_JSON='{"base": ["SPP_KC_COLD_LOOP=0"], "cold_loop": ["SPP_KC_COLD_LOOP=1"]}' VARIANT_DEEPCAM=0 \
  VARIANT_SWEEP="lam2.0_rho0.7,lam2.0_rho0.0,lam16.0_rho0.9,lam16.0_rho0.0,lam64.0_rho0.7" \
  timeout 2400 python scripts/variants.py run > gpurun_out/r02v_kc_cold_loop.log 2>&1
echo done
