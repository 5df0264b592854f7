#!/usr/bin/env bash
# KL 4-row groups (8 lanes per row, <= 8 runs), pairs and single rows as fallbacks: label tests, bench x2, ncu
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_labels.py -q -x > gpurun_out/r02b8_labels_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r02b8_labels_pytest.log
timeout 600 python scripts/label_bench.py > gpurun_out/r02b8_label_bench.json 2> gpurun_out/r02b8_label_bench.err
timeout 600 python scripts/label_bench.py > gpurun_out/r02b8_label_bench_rep2.json 2>> gpurun_out/r02b8_label_bench.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kl_decode_mask -s 3 -c 1 -o gpurun_out/r02b8_kl python scripts/label_bench.py > gpurun_out/r02b8_kl_ncu.log 2>&1
echo done
