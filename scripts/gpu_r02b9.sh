#!/usr/bin/env bash
# KL row groups: 4-row groups at 3/4/5 CTAs per SM (79/64/48 registers) vs pairs only (4/5 CTAs), label bench x2
set -u
mkdir -p gpurun_out
for rep in 1 2; do
for v in q4 q5 q3 pairs4 pairs5; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python scripts/label_bench.py > gpurun_out/r02b9_label_bench_${v}_rep$rep.json 2>> gpurun_out/r02b9_label_bench.err
done
done
echo done
