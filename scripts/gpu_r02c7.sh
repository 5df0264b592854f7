#!/usr/bin/env bash
# KC: L2 evict_last policy created by a pure asm (rematerialisable) vs volatile; cosmo parity
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_limits.py -q -x -k "cosmo" > gpurun_out/r02c7_pytest_cosmo.log 2>&1; echo "rc=$?" >> gpurun_out/r02c7_pytest_cosmo.log
export VARIANT_DEEPCAM=0 VARIANT_SWEEP=lam16.0_rho0.9,lam2.0_rho0.0,lam2.0_rho0.7
for rep in 1 2 3; do
timeout 1200 python scripts/variants.py run > gpurun_out/r02c7_kc_polpure_rep$rep.log 2>&1
done
echo done
