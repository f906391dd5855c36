# session-5b: interior-body parity test, bench with the busy pre-roll (K=1000 x3 + default line)
timeout 900 python -m pytest tests/test_gpu_parity.py -k interior_fast_body -q -x --timeout 600 > gpurun_out/pytest_s5b.log 2>&1; tail -2 gpurun_out/pytest_s5b.log
for r in 1 2 3; do
  timeout 300 python bench.py --config C2 --precision fp64 --steps 1000 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_s5b.jsonl 2>> gpurun_out/bench_s5b.err
done
timeout 300 python bench.py --config C2 --precision fp32 --steps 1000 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_s5b.jsonl 2>> gpurun_out/bench_s5b.err
timeout 600 python bench.py > gpurun_out/bench_default_s5b.json 2> gpurun_out/bench_default_s5b.err
python tools/show_bench.py gpurun_out/bench_s5b.jsonl gpurun_out/bench_default_s5b.json; tail -3 gpurun_out/bench_s5b.err
