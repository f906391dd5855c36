# 3D boundary-free body (MRLBM_FAST_PATH_3D) vs the default build: parity of the variant + A/B on C3/C4/C5w
MRLBM_LIB=$PWD/ab/libmrlbm_f3.so timeout 600 python -m pytest tests/test_gpu_parity.py -k "D3Q" -q -x --timeout 300 > gpurun_out/pytest_f3.log 2>&1; tail -2 gpurun_out/pytest_f3.log
LIBS="f3=ab/libmrlbm_f3.so D=" STEPS=600 bash tools/abn.sh f3 "C3 fp64" "C4 fp32" "C5 fp64" > /dev/null
cat gpurun_out/ab_f3.txt
