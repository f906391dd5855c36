# rotated sweep (pulls of layer it interleaved with the collision of layer it+1) in the scalar kernel
MRLBM_LIB=$PWD/ab/libmrlbm_rot.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py tests/test_gpu_slabs.py -m gpu -q -x -k "D2Q9 or D3Q19 or 2d" > gpurun_out/ab10_pytest_rot.log 2>&1; tail -n 2 gpurun_out/ab10_pytest_rot.log
bash tools/ab_libs.sh ab10 "cur rot" "C3 fp64" "C5 fp64" "C2 fp64" "C2 fp32"
