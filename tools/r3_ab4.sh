MRLBM_TILE=11 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -m gpu -q -x -k "D3Q or 3d or 3D" > gpurun_out/ab4_pytest_t11.log 2>&1; tail -2 gpurun_out/ab4_pytest_t11.log
MRLBM_TILE=12 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "D3Q27" > gpurun_out/ab4_pytest_t12.log 2>&1; tail -2 gpurun_out/ab4_pytest_t12.log
bash tools/ab_libs.sh ab4 "cur cur:MRLBM_TILE=10 cur:MRLBM_TILE=11 cur:MRLBM_TILE=12 cur:MRLBM_TILE=9" "C4 fp32" "C5 fp64" "C3 fp64"
