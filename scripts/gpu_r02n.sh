#!/usr/bin/env bash
# KCX (dense-sample cluster kernel, profiles/r02n_kcx_dsmem_experiment.patch): parity, then A/B against the build without it; run twice (hot-group duplication layout; 8-group interleave, with r02n_ renamed r02o_)
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "dense_cluster" -s > gpurun_out/r02n_kcx_parity.log 2>&1; echo "rc=$?" >> gpurun_out/r02n_kcx_parity.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "cosmo" > gpurun_out/r02n_cosmo_parity.log 2>&1; echo "rc=$?" >> gpurun_out/r02n_cosmo_parity.log
ONLY="lam2.0_rho0.7,lam2.0_rho0.0,lam16.0_rho0.9,lam16.0_rho0.0,lam64.0_rho0.7,lam64.0_rho0.0"
for v in kcx_on kcx_off kcx_on kcx_off; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python scripts/sweep.py --pool 2 --steps 10 --policies default --only $ONLY > gpurun_out/r02n_sweep_$v.json 2>> gpurun_out/r02n_sweep.err
done
for v in kcx_on kcx_off; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python bench.py --steps 20 --warmup 5 --e2e-steps 2 --cpu-seconds 0.5 --secondary none > gpurun_out/r02n_bench_$v.json 2>> gpurun_out/r02n_bench.err
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python scripts/big_volume.py > gpurun_out/r02n_big_$v.json 2>> gpurun_out/r02n_big.err
done
echo done
