# r02: physics validation (tools/csr_validation.py): forces vs the semi-analytic steady state and
# the 1D CSR line charge at 129^2, and the Monte-Carlo MSE vs N (Fig. 3)
set -x
timeout 900 python tools/csr_validation.py 129 --out gpurun_out/r02_csr_forces_129.json > gpurun_out/csr_forces.log 2>&1; tail -3 gpurun_out/csr_forces.log | cut -c1-1500
timeout 1500 python tools/csr_validation.py --mse --out gpurun_out/r02_csr_mse.json > gpurun_out/csr_mse.log 2>&1; tail -3 gpurun_out/csr_mse.log | cut -c1-1500
