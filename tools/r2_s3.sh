# round-2 session 3: GPU suite after the staging change, 2D wave-fill sweep, C5 1024^3 on one GPU
mkdir -p gpurun_out
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s3_smoke.log 2>&1 || { echo smoke failed; tail -5 gpurun_out/r2s3_smoke.log; exit 1; }
timeout 1200 python -m pytest tests -q -m gpu --timeout 300 -x > gpurun_out/r2s3_pytest.log 2>&1; tail -3 gpurun_out/r2s3_pytest.log
bash tools/seg2d.sh seg2d_r2s3 > gpurun_out/seg2d_r2s3.txt 2>&1; cat gpurun_out/seg2d_r2s3.txt
free -g | head -2
timeout 1200 python bench.py --config C5 --strong --steps 40 --warmup 4 --no-cpu-baseline --no-e2e > gpurun_out/r2s3_c5strong1.json 2> gpurun_out/r2s3_c5strong1.err; python tools/show_bench.py gpurun_out/r2s3_c5strong1.json; tail -3 gpurun_out/r2s3_c5strong1.err
