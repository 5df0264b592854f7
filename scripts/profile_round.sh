#!/usr/bin/env bash
# Round profiling on the GPU box (run under gpurun; one GPU):
#   1. launch list of the bench command (ncu gpu__time_duration, cold-cache, serialised)
#   2. ncu --set full of the dominant kernels (KC for C2, KD for C4)
# Outputs land in gpurun_out/; summarise here with scripts/ncu_summary.py and
# scripts/launch_summary.py into profiles/.
set -u
R=${1:-r02}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${R}_launches.csv \
    python bench.py --steps 20 --warmup 3 --e2e-steps 1 --cpu-seconds 1 --secondary none \
    > gpurun_out/${R}_launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:kc_expand -s 3 -c 1 -o gpurun_out/${R}_kc \
    python bench.py --steps 2 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 --secondary none \
    > gpurun_out/${R}_kc_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:kd_decode -s 3 -c 1 -o gpurun_out/${R}_kd \
    python bench.py --workload deepcam --steps 2 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 \
    > gpurun_out/${R}_kd_ncu.log 2>&1
echo done
ncu --set full --clock-control none --import-source on -k regex:kc_expand -s 3 -c 1 -o gpurun_out/${R}_kc_esc \
    python bench.py --steps 2 --warmup 3 --e2e-steps 1 --cpu-seconds 0.2 --secondary none --escape-keys \
    > gpurun_out/${R}_kc_esc_ncu.log 2>&1
echo done-esc
