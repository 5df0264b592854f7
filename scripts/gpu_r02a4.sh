#!/usr/bin/env bash
# RAW-slab path rewrite: cosmo GPU parity; KD line-load evict_first A/B; C5 RAW rows
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k cosmo > gpurun_out/r02a4_pytest_cosmo.log 2>&1; echo "rc=$?" >> gpurun_out/r02a4_pytest_cosmo.log
timeout 600 python scripts/sweep.py --pool 2 --steps 10 --only lam64.0_rho0.0,lam2.0_rho0.0,lam16.0_rho0.9 > gpurun_out/r02a4_sweep_raw.json 2> gpurun_out/r02a4_sweep_raw.err
export VARIANT_COSMO=0
for rep in 1 2; do
timeout 900 python scripts/variants.py run > gpurun_out/r02a4_kd_line_ef_rep$rep.log 2>&1
done
echo done
