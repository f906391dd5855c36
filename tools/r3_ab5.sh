# p7: halo-row specialisation in the paired kernel; old kernel with the regrouped D3Q19 collision
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -m gpu -q -x -k "D3Q or 3d or 3D" > gpurun_out/ab5_pytest_t0.log 2>&1; tail -2 gpurun_out/ab5_pytest_t0.log
MRLBM_TILE=9 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "D3Q19" > gpurun_out/ab5_pytest_t9.log 2>&1; tail -2 gpurun_out/ab5_pytest_t9.log
MRLBM_TILE=11 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "D3Q" > gpurun_out/ab5_pytest_t11.log 2>&1; tail -2 gpurun_out/ab5_pytest_t11.log
bash tools/ab_libs.sh ab5 "p5 cur cur:MRLBM_TILE=9 cur:MRLBM_TILE=10 cur:MRLBM_TILE=11" "C4 fp32" "C5 fp64" "C3 fp64"
