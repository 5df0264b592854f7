#!/usr/bin/env bash
# KC L2-policy variants (key evict_first, cold evict_last, tail normal / demoted): timing x2 + ncu DRAM bytes
set -u
mkdir -p gpurun_out
export VARIANT_DEEPCAM=0
for rep in 1 2; do
timeout 900 python scripts/variants.py run > gpurun_out/r02a3_kc_l2policy_rep$rep.log 2>&1
done
for v in base key_ef cold_el tail_norm tail_demote all3; do
  SPP_LIB=paper_conf_ipps_ibrahimo22_b200/variants/libspp_$v.so timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum --clock-control none -k regex:kc_expand -s 6 -c 2 --csv python bench.py --secondary none --steps 3 --warmup 3 --cpu-seconds 0.5 --e2e-steps 1 > gpurun_out/r02a3_ncu_$v.csv 2>/dev/null
done
echo done
