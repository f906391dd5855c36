# PUSH-template build: parity + A/B against the pre-P2P build (fd) and the 3D fast-path build (f3)
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_slabs.py tests/test_gpu_p2p.py tests/test_gpu_fd.py -q -x --timeout 300 > gpurun_out/pytest_push.log 2>&1; tail -2 gpurun_out/pytest_push.log
MRLBM_LIB=$PWD/ab/libmrlbm_f3.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_p2p.py -q -x --timeout 300 > gpurun_out/pytest_pushf3.log 2>&1; tail -2 gpurun_out/pytest_pushf3.log
LIBS="fd=ab/libmrlbm_fd.so E=" STEPS=800 bash tools/abn.sh push "C2 fp64" "C2 fp32" > /dev/null
LIBS="fd=ab/libmrlbm_fd.so E= f3=ab/libmrlbm_f3.so" STEPS=500 bash tools/abn.sh push "C3 fp64" "C4 fp32" "C5 fp64" > /dev/null
cat gpurun_out/ab_push.txt
