#!/usr/bin/env bash
# KC C2 DRAM/L2 traffic attribution with the key evict_first hint: main launch (-s 3 -c 1)
set -u
mkdir -p gpurun_out
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_op_write.sum
for v in base notail nocold; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 300 ncu --metrics $M --clock-control none -k regex:kc_expand -s 3 -c 1 --csv python bench.py --secondary none --steps 2 --warmup 3 --cpu-seconds 0.2 --e2e-steps 1 > gpurun_out/r02a7_ncu_$v.csv 2>/dev/null
done
export VARIANT_DEEPCAM=0
timeout 900 python scripts/variants.py run > gpurun_out/r02a7_variants.log 2>&1
echo done
