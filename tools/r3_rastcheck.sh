# grouped launch order: parity with forced (ragged) groups on small grids, full-size C5 slab, default suite pieces
MRLBM_RAST=3 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py -m gpu -q -x -k "D3Q" > gpurun_out/rast3_pytest.log 2>&1; tail -n 1 gpurun_out/rast3_pytest.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_slabs.py tests/test_gpu_p2p.py -m gpu -q -x > gpurun_out/rastdef_pytest.log 2>&1; tail -n 1 gpurun_out/rastdef_pytest.log
timeout 300 python bench.py --config C5 --steps 200 --no-cpu-baseline --no-e2e > gpurun_out/bench_r03_c5rast.json 2>/dev/null; python tools/show_bench.py gpurun_out/bench_r03_c5rast.json
