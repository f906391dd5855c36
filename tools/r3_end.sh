# end-of-round check of the committed state: GPU suite, smoke, default bench line (with cpu baseline and e2e)
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_r03_end.log 2>&1; tail -n 1 gpurun_out/pytest_r03_end.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r03_end.log 2>&1; tail -n 1 gpurun_out/smoke_r03_end.log
timeout 600 python bench.py > gpurun_out/bench_r03_end_default.json 2>/dev/null; python tools/show_bench.py gpurun_out/bench_r03_end_default.json
