#!/usr/bin/env bash
# round-2 GPU session c: full GPU suite (labels, limits), racecheck reproducer, KC cold-path variants
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02c_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02c_pytest_gpu.log
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_repro.cu
for v in 0 1 2 3; do timeout 300 compute-sanitizer --tool racecheck /tmp/rr $v > gpurun_out/r02c_racecheck_repro_v$v.log 2>&1; done
VARIANT_DEEPCAM=0 VARIANT_SWEEP="lam2.0_rho0.7,lam16.0_rho0.9,lam16.0_rho0.7,lam64.0_rho0.7" VARIANTS_JSON='{"base": [], "kc_fixup": ["SPP_KC_FIXUP=1"], "kc_la2": ["SPP_KC_LA=2", "SPP_KC_HOT_KB=120"], "kc_fixup_la2": ["SPP_KC_FIXUP=1", "SPP_KC_LA=2", "SPP_KC_HOT_KB=120"]}' timeout 2400 python scripts/variants.py run > gpurun_out/r02c_variants.log 2>&1
echo done
