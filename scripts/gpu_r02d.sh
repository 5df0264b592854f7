#!/usr/bin/env bash
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02d_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02d_pytest_gpu.log
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_repro.cu
for v in 3 4 5; do timeout 300 compute-sanitizer --tool racecheck /tmp/rr $v > gpurun_out/r02d_racecheck_repro_v$v.log 2>&1; done
for c in deepcam_default deepcam_bigline; do timeout 900 compute-sanitizer --tool racecheck python scripts/sanitize_fullsize.py $c > gpurun_out/r02d_racecheck_$c.log 2>&1; done
echo done
