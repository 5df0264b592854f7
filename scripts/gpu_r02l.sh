#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_labels.py tests/test_bench_contract.py -q > gpurun_out/r02l_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02l_pytest.log
timeout 600 python scripts/label_bench.py > gpurun_out/r02l_label_bench.json 2>&1
for rep in 1 2; do
VARIANT_DEEPCAM=0 VARIANTS_JSON='{"base": [], "kc_nopf": ["SPP_KC_PREFETCH_TAIL=0"], "kc_wb": ["SPP_STORE_CS=0"]}' timeout 1500 python scripts/variants.py run > gpurun_out/r02l_variants_rep$rep.log 2>&1
done
echo done
