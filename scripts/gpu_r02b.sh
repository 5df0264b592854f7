#!/usr/bin/env bash
# round-2 GPU session b: GPU suite, KC dense-slab slots and KD variants, racecheck, C5 + big volumes
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02b_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02b_pytest_gpu.log
VARIANT_SWEEP="lam2.0_rho0.7,lam2.0_rho0.0,lam16.0_rho0.9,lam16.0_rho0.7,lam64.0_rho0.9,lam64.0_rho0.7" VARIANTS_JSON='{"base": [], "kc_dense0": ["SPP_KC_DENSE=0"], "kd_reacq0": ["SPP_KD_PROD_REACQUIRE=0"], "kd_slot2432": ["SPP_KD_WS_SLOT=2432"]}' timeout 2400 python scripts/variants.py run > gpurun_out/r02b_variants.log 2>&1
timeout 1500 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py deepcam > gpurun_out/r02b_racecheck_deepcam.log 2>&1
timeout 900 python scripts/big_volume.py > gpurun_out/r02b_big_volume.json 2> gpurun_out/r02b_big_volume.err
SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_kc_dense0.so timeout 900 python scripts/big_volume.py > gpurun_out/r02b_big_volume_dense0.json 2>&1
echo done
