#!/usr/bin/env bash
# KD four prefix chains per lane (vs two): DeepCAM parity + limits, alternating C4 bench A/B, ncu of KD
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_limits.py -q -k "deepcam or line or raw or limit or mode" > gpurun_out/r02t_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02t_pytest.log
for rep in 1 2 3; do
  for lib in paper_conf_ipps_ibrahimo22_b200/variants/libspp_kd_chains2.so paper_conf_ipps_ibrahimo22_b200/libspp.so; do
    SPP_LIB=$lib timeout 600 python bench.py --workload deepcam --steps 20 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 > gpurun_out/r02t_kd_$(basename $lib .so)_$rep.json 2>/dev/null
  done
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kd_decode -s 3 -c 1 -o gpurun_out/r02t_kd python bench.py --workload deepcam --steps 2 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 > gpurun_out/r02t_kd_ncu.log 2>&1
echo done
