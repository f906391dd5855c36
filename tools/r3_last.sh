# final check of the pruned build: GPU suite, smoke, default bench line
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_r03z.log 2>&1; tail -n 2 gpurun_out/pytest_r03z.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r03z.log 2>&1; tail -n 1 gpurun_out/smoke_r03z.log
timeout 600 python bench.py > gpurun_out/bench_r03z_default.json 2> gpurun_out/bench_r03z_default.err; python tools/show_bench.py gpurun_out/bench_r03z_default.json
for cfg in "C4 fp32" "C5 fp64" "C3 fp64"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline >> gpurun_out/bench_r03z_side.jsonl 2>/dev/null
done
python tools/show_bench.py gpurun_out/bench_r03z_side.jsonl
