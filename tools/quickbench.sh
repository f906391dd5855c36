# usage: bash tools/quickbench.sh TAG  -- parity tests + bench lines for C2/C3/C4 (no CPU baseline)
TAG=$1
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_$TAG.log 2>&1; tail -2 gpurun_out/pytest_$TAG.log
for cfg in "C2 fp64" "C2 fp32" "C3 fp64" "C4 fp32" "C4 fp64"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-1000} --warmup 20 --no-cpu-baseline >> gpurun_out/bench_$TAG.jsonl 2>> gpurun_out/bench_$TAG.err
done
python tools/show_bench.py gpurun_out/bench_$TAG.jsonl
