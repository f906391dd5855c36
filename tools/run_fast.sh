# fast-path (boundary-free body for interior CTAs) parity + A/B against the pre-P2P (fd) and P2P (B) builds
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_slabs.py tests/test_gpu_p2p.py tests/test_gpu_fd.py -q -x --timeout 300 > gpurun_out/pytest_fast.log 2>&1; tail -2 gpurun_out/pytest_fast.log
MRLBM_LIB=$PWD/ab/libmrlbm_f3.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_slabs.py tests/test_gpu_fd.py -q -x --timeout 300 > gpurun_out/pytest_f3.log 2>&1; tail -2 gpurun_out/pytest_f3.log
LIBS="fd=ab/libmrlbm_fd.so B=ab/libmrlbm_B.so D=" STEPS=1000 bash tools/abn.sh fast "C2 fp64" "C2 fp32" > /dev/null
LIBS="fd=ab/libmrlbm_fd.so B=ab/libmrlbm_B.so f3=ab/libmrlbm_f3.so" STEPS=600 bash tools/abn.sh fast "C3 fp64" "C4 fp32" "C5 fp64" > /dev/null
cat gpurun_out/ab_fast.txt
