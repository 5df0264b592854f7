#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_repro.cu
for v in 4 5 6; do for k in 1 2 3; do timeout 300 compute-sanitizer --tool racecheck /tmp/rr $v > gpurun_out/r02e_racecheck_repro_v${v}_run$k.log 2>&1; done; done
VARIANT_DEEPCAM=0 VARIANT_SWEEP="lam2.0_rho0.7,lam16.0_rho0.9,lam16.0_rho0.7,lam64.0_rho0.9,lam64.0_rho0.7" VARIANTS_JSON='{"base": [], "kc_pfl1": ["SPP_KC_PF_L1=1"]}' timeout 2400 python scripts/variants.py run > gpurun_out/r02e_variants.log 2>&1
SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_kc_pfl1.so timeout 900 python scripts/big_volume.py > gpurun_out/r02e_big_volume_pfl1.json 2>&1
timeout 900 python scripts/big_volume.py > gpurun_out/r02e_big_volume_base.json 2>&1
echo done
