# re-measure the ST C2 baseline (session-5 reading 34.1k vs 44.2k in session 4) and MR C2 on one box
for r in 1 2 3; do for m in ST MR; do
  timeout 300 python bench.py --config C2 --precision fp64 --method $m --steps 1000 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_strecheck.jsonl 2>> gpurun_out/bench_strecheck.err
done; done
python tools/show_bench.py gpurun_out/bench_strecheck.jsonl
