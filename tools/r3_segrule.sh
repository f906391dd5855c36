# segment rule with a 4-layer overhead term vs the previous choice (64 layers for C4 / C5w, 86 for C3)
bash tools/ab_libs.sh ab16 "cur cur:MRLBM_SEG=64" "C4 fp32" "C5 fp64"
timeout 300 python bench.py --config C3 --steps 200 --no-cpu-baseline --no-e2e | python tools/show_bench.py /dev/stdin
timeout 600 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_parity.py -m gpu -q -x -k "D3Q27 or C4 or fullsize" > gpurun_out/segrule_pytest.log 2>&1; tail -n 1 gpurun_out/segrule_pytest.log
