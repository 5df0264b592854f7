#!/usr/bin/env bash
# KD producer back-off 100 / 400 / 1000 ns under sustained load (power trace) and in the C4 bench
set -u
mkdir -p gpurun_out
for rep in 1 2; do
for v in sl100 sl400 sl1000; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 600 python scripts/kd_power_trace.py > gpurun_out/r02c6_kd_trace_${v}_rep$rep.json 2>> gpurun_out/r02c6.err
done
done
echo done
