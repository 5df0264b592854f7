#!/usr/bin/env bash
# KL: 8 CTAs per SM (two waves) with and without the evict_first row-store hint
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_labels.py -q -x > gpurun_out/r02b3_labels_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02b3_labels_pytest.log
for rep in 1 2; do
for v in kl_base8 kl_ef8; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python scripts/label_bench.py > gpurun_out/r02b3_label_bench_${v}_rep$rep.json 2>> gpurun_out/r02b3_label_bench.err
done
done
echo done
