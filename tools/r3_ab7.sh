# p8: product-form D3Q27-R collide+reconstruct in the paired kernel; one-body variants (tiles 13/14)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -m gpu -q -x -k "D3Q27" > gpurun_out/ab7_pytest_t0.log 2>&1; tail -n 2 gpurun_out/ab7_pytest_t0.log
MRLBM_TILE=10 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "D3Q27" > gpurun_out/ab7_pytest_t10.log 2>&1; tail -n 2 gpurun_out/ab7_pytest_t10.log
MRLBM_TILE=13 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "D3Q" > gpurun_out/ab7_pytest_t13.log 2>&1; tail -n 2 gpurun_out/ab7_pytest_t13.log
bash tools/ab_libs.sh ab7 "p6 cur cur:MRLBM_TILE=9 cur:MRLBM_TILE=10 cur:MRLBM_TILE=11 cur:MRLBM_TILE=13 cur:MRLBM_TILE=14" "C4 fp32" "C5 fp64" "C3 fp64"
