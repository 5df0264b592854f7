#!/usr/bin/env bash
# sanitizers on the final code
set -u
mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool memcheck python scripts/sanitize_cases.py > gpurun_out/r02m_memcheck_cases.log 2>&1
timeout 900 compute-sanitizer --tool synccheck python scripts/sanitize_cases.py > gpurun_out/r02m_synccheck_cases.log 2>&1
timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize_cases.py > gpurun_out/r02m_racecheck_cases.log 2>&1
for c in deepcam_default deepcam_bigline deepcam_long; do timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py $c > gpurun_out/r02m_racecheck_$c.log 2>&1; done
for c in deepcam deepcam_long cosmo; do timeout 1200 compute-sanitizer --tool memcheck python scripts/sanitize_fullsize.py $c > gpurun_out/r02m_memcheck_full_$c.log 2>&1; done
timeout 1200 compute-sanitizer --tool synccheck python scripts/sanitize_fullsize.py deepcam > gpurun_out/r02m_synccheck_full_deepcam.log 2>&1
echo done
