#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_limits.py tests/test_gpu_labels.py tests/test_loader.py -q > gpurun_out/r02j_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02j_pytest.log
for rep in 1 2 3; do
  for lib in paper_conf_ipps_ibrahimo22_b200/variants/libspp_kd_before.so paper_conf_ipps_ibrahimo22_b200/libspp.so; do
    SPP_LIB=$lib timeout 600 python bench.py --workload deepcam --steps 20 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 > gpurun_out/r02j_kd_$(basename $lib .so)_$rep.json 2>/dev/null
  done
done
timeout 600 python scripts/label_bench.py > gpurun_out/r02j_label_bench.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kl_decode_mask -s 3 -c 1 -o gpurun_out/r02j_kl python scripts/label_bench.py > gpurun_out/r02j_kl_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kd_decode -s 3 -c 1 -o gpurun_out/r02j_kd python bench.py --workload deepcam --steps 2 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 > gpurun_out/r02j_kd_ncu.log 2>&1
echo done
