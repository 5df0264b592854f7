#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_limits.py tests/test_gpu_labels.py -q > gpurun_out/r02g_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02g_pytest.log
for rep in 1 2; do
VARIANT_COSMO=0 VARIANTS_JSON='{"base": [], "kd_ns3_s1216": ["SPP_KD_WS_SLOT=1216"], "kd_ns4_s1216": ["SPP_KD_WS_NS=4", "SPP_KD_WS_SLOT=1216"], "kd_ns5_s1216": ["SPP_KD_WS_NS=5", "SPP_KD_WS_SLOT=1216"], "kd_ns4_s1536": ["SPP_KD_WS_NS=4", "SPP_KD_WS_SLOT=1536"]}' timeout 1500 python scripts/variants.py run > gpurun_out/r02g_variants_rep$rep.log 2>&1
done
echo done
