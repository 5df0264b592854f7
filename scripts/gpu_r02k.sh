#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -k cosmo > gpurun_out/r02k_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02k_pytest.log
for rep in 1 2 3; do
  for lib in paper_conf_ipps_ibrahimo22_b200/variants/libspp_kc_before.so paper_conf_ipps_ibrahimo22_b200/variants/libspp_kc_stagepos.so; do
    SPP_LIB=$lib timeout 600 python bench.py --steps 100 --warmup 10 --secondary none --e2e-steps 1 --cpu-seconds 0.2 > gpurun_out/r02k_kc_$(basename $lib .so)_$rep.json 2>/dev/null
  done
done
echo done
