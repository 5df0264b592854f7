#!/usr/bin/env bash
# KC: the third cold key's LUT row loaded before the expansion loop (ovf) vs in the loop (base); cosmo parity
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam16.0_rho0.9,lam16.0_rho0.7,lam64.0_rho0.7,lam2.0_rho0.0
for rep in 1 2; do
timeout 1500 python scripts/variants.py run > gpurun_out/r02c5_kc_ovf_rep$rep.log 2>&1
done
SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_ovf.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "cosmo" > gpurun_out/r02c5_pytest_cosmo_ovf.log 2>&1; echo "rc=$?" >> gpurun_out/r02c5_pytest_cosmo_ovf.log
echo done
