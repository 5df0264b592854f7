#!/usr/bin/env bash
# KL staged RUN rows: label parity, label bench, ncu of KL
set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_labels.py -q > gpurun_out/r02p_labels_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02p_labels_pytest.log
timeout 600 python scripts/label_bench.py > gpurun_out/r02p_label_bench.json 2> gpurun_out/r02p_label_bench.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kl_decode_mask -s 3 -c 1 -o gpurun_out/r02p_kl python scripts/label_bench.py > gpurun_out/r02p_kl_ncu.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_labels.py -q -k lossless > gpurun_out/r02p_labels_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02p_labels_memcheck.log
echo done
