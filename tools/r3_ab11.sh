# scalar-kernel rotation now default in 3D; paired-kernel rotation (rp) A/B; D3Q27 / D3Q19-fp32 parity with rp
MRLBM_LIB=$PWD/ab/libmrlbm_rp.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -m gpu -q -x -k "D3Q27 or fp32" > gpurun_out/ab11_pytest_rp.log 2>&1; tail -n 2 gpurun_out/ab11_pytest_rp.log
bash tools/ab_libs.sh ab11 "p11 cur rp" "C4 fp32" "C3 fp32" "C5 fp32" "C5 fp64" "C4 fp64"
