# round 2 session 2: full GPU suite + smoke + default bench + C5w bench
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r2s2_pytest.log 2>&1; tail -3 gpurun_out/r2s2_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s2_smoke.log 2>&1; tail -1 gpurun_out/r2s2_smoke.log
timeout 900 python bench.py > gpurun_out/r2s2_bench_default.json 2> gpurun_out/r2s2_bench_default.err; tail -c 400 gpurun_out/r2s2_bench_default.err
timeout 600 python bench.py --config C5 --no-cpu-baseline --steps 200 > gpurun_out/r2s2_bench_c5.json 2> gpurun_out/r2s2_bench_c5.err
python tools/show_bench.py gpurun_out/r2s2_bench_default.json gpurun_out/r2s2_bench_c5.json
