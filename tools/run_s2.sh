timeout 600 python -m pytest tests/test_gpu_parity.py -q -x --timeout 600 > gpurun_out/pytest_s2.log 2>&1; tail -1 gpurun_out/pytest_s2.log
LIBS="noh=ab/libmrlbm_noh.so B=" STEPS=600 bash tools/abn.sh s2h "C3 fp64" "C4 fp32" > /dev/null
STEPS=600 TILES="0 1 2 3" bash tools/sweep.sh s2t "C2 fp64" > /dev/null
STEPS=400 TILES="1 2" bash tools/sweep.sh s2t3 "C3 fp64" "C5 fp64" > /dev/null
cat gpurun_out/ab_s2h.txt gpurun_out/sweep_s2t.txt gpurun_out/sweep_s2t3.txt
