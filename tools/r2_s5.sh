# round-2 session 5: 2D segment default 12 (fp64) / 16 (fp32): tests, bench lines, ncu of C2
mkdir -p gpurun_out
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s5_smoke.log 2>&1 || { echo smoke failed; exit 1; }
timeout 1200 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/r2s5_pytest.log 2>&1; tail -3 gpurun_out/r2s5_pytest.log
timeout 600 python bench.py > gpurun_out/r2s5_default.json 2> gpurun_out/r2s5_default.err
timeout 300 python bench.py --config C2 --precision fp32 > gpurun_out/r2s5_c2fp32.json 2> gpurun_out/r2s5_c2fp32.err
timeout 300 python bench.py --steps 20 --warmup 3 > gpurun_out/r2s5_k20.json 2> gpurun_out/r2s5_k20.err
python tools/show_bench.py gpurun_out/r2s5_default.json gpurun_out/r2s5_c2fp32.json gpurun_out/r2s5_k20.json
bash tools/ncu_capture.sh r02s5 "C2 fp64" "C2 fp32" > /dev/null 2>&1
ls gpurun_out | grep r02s5
