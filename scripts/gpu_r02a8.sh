#!/usr/bin/env bash
# KD: decoded-row TMA bulk stores with an L2 evict_first hint vs plain (C4, 3 alternating reps)
set -u
mkdir -p gpurun_out
export VARIANT_COSMO=0
for rep in 1 2 3; do
timeout 900 python scripts/variants.py run > gpurun_out/r02a8_kd_row_ef_rep$rep.log 2>&1
done
echo done
