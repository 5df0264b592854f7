#!/usr/bin/env bash
# round-2 final evidence on the end-of-round code: GPU suite, smoke, bench line, reference
# arm, C5 sweep, larger volumes, single samples, labels, launch list + ncu captures
set -u
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02end2_final_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02end2_final_pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02end2_final_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02end2_final_smoke.log
timeout 900 python bench.py > gpurun_out/r02end2_final_bench.json 2> gpurun_out/r02end2_final_bench.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02end2_final_ref.json 2> gpurun_out/r02end2_final_ref.err
timeout 1500 python scripts/sweep.py --pool 2 --steps 10 > gpurun_out/r02end2_c5_sweep.json 2> gpurun_out/r02end2_c5_sweep.err
timeout 900 python scripts/big_volume.py > gpurun_out/r02end2_big_volume.json 2> gpurun_out/r02end2_big_volume.err
timeout 900 python scripts/single_sample.py > gpurun_out/r02end2_single_sample.json 2> gpurun_out/r02end2_single_sample.err
timeout 600 python scripts/label_bench.py > gpurun_out/r02end2_label_bench.json 2> gpurun_out/r02end2_label_bench.err
timeout 2400 bash scripts/profile_round.sh r02end2 > gpurun_out/r02end2_profile_round.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:kl_decode_mask -s 3 -c 1 -o gpurun_out/r02end2_kl python scripts/label_bench.py > gpurun_out/r02end2_kl_ncu.log 2>&1
echo done
timeout 800 python scripts/kd_power_trace.py > gpurun_out/r02end2_kd_power_trace.json 2> gpurun_out/r02end2_kd_power_trace.err
