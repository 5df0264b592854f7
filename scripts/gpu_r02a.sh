#!/usr/bin/env bash
# round-2 GPU session a: full GPU suite, default bench, KD slot variants, sanitizers
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02a_smi.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/r02a_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02a_pytest_gpu.log
timeout 900 python bench.py > gpurun_out/r02a_bench.json 2> gpurun_out/r02a_bench.err; echo "bench rc=$?"
VARIANT_COSMO=0 VARIANTS_JSON='{"kd_slot2048": [], "kd_slot2304": ["SPP_KD_WS_SLOT=2304"], "kd_slot2432": ["SPP_KD_WS_SLOT=2432"], "kd_slot1792": ["SPP_KD_WS_SLOT=1792"]}' timeout 900 python scripts/variants.py run > gpurun_out/r02a_variants.log 2>&1
timeout 1500 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py deepcam > gpurun_out/r02a_racecheck_deepcam.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize_fullsize.py deepcam_long > gpurun_out/r02a_memcheck_deepcam_long.log 2>&1
timeout 600 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py deepcam_long > gpurun_out/r02a_racecheck_deepcam_long.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python scripts/sanitize_cases.py > gpurun_out/r02a_memcheck_cases.log 2>&1
echo done
