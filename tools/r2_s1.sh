# round 2 session 1: long 3D parity + ST tolerance + ncu source captures of the 3D kernels
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.max.sm --format=csv > gpurun_out/r2s1_gpu.txt
timeout 1500 python -m pytest tests/test_gpu_parity_long.py tests/test_gpu_st.py -q -m gpu > gpurun_out/r2s1_pytest.log 2>&1; tail -5 gpurun_out/r2s1_pytest.log
NO_LAUNCHES=1 bash tools/ncu_capture.sh r02s1 "C3 fp64" "C4 fp32" "C5 fp64" > /dev/null 2>&1
ls gpurun_out
