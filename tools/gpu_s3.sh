TAG=$1
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log
STEPS=600 bash tools/ab.sh $TAG "C2 fp64" "C2 fp32" "C3 fp64" "C4 fp32"
for cfg in "C2 fp64 ST" "C2 fp32 ST" "C3 fp64 ST" "C4 fp32 ST"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --method $3 --steps 300 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_st_$TAG.jsonl 2>> gpurun_out/bench_st_$TAG.err
done
python tools/show_bench.py gpurun_out/bench_st_$TAG.jsonl
