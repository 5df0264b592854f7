#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_repro.cu
for v in 7 8; do for k in 1 2; do timeout 300 compute-sanitizer --tool racecheck /tmp/rr $v > gpurun_out/r02f_racecheck_repro_v${v}_run$k.log 2>&1; done; done
VARIANT_COSMO=0 VARIANTS_JSON='{"base": [], "kd_serial": ["SPP_KD_PROD_SERIAL=1"]}' timeout 1200 python scripts/variants.py run > gpurun_out/r02f_variants.log 2>&1
VARIANT_COSMO=0 VARIANTS_JSON='{"base": [], "kd_serial": ["SPP_KD_PROD_SERIAL=1"]}' timeout 1200 python scripts/variants.py run > gpurun_out/r02f_variants_rep2.log 2>&1
for c in deepcam_bigline deepcam_default; do SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_kd_serial.so timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py $c > gpurun_out/r02f_racecheck_serial_$c.log 2>&1; done
timeout 600 python scripts/kd_instance_ab.py > gpurun_out/r02f_kd_instance_ab.json 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02f_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02f_pytest_gpu.log
echo done
