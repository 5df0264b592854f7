#!/usr/bin/env bash
# KD: row-store policy chosen per launch (evict_first above 64 MB of output, normal below):
# DeepCAM parity, C3 single-sample latency, C4 bench line x2
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_limits.py -q -x -k "deepcam or host_pipeline or loader" > gpurun_out/r02b5_pytest_deepcam.log 2>&1; echo "rc=$?" >> gpurun_out/r02b5_pytest_deepcam.log
timeout 900 python scripts/single_sample.py > gpurun_out/r02b5_single_sample.json 2> gpurun_out/r02b5_single_sample.err
for rep in 1 2; do
timeout 600 python bench.py --workload deepcam --steps 20 --warmup 3 --e2e-steps 1 --cpu-seconds 0.5 > gpurun_out/r02b5_bench_c4_rep$rep.json 2>> gpurun_out/r02b5_bench.err
done
echo done
