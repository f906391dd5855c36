# usage: bash tools/gpu_check.sh TAG -- GPU parity tests, smoke, MR + ST bench lines (no CPU baseline)
TAG=$1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi_$TAG.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
for cfg in "C2 fp64 MR" "C2 fp32 MR" "C3 fp64 MR" "C4 fp32 MR" "C2 fp64 ST" "C3 fp64 ST" "C4 fp32 ST"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --method $3 --steps ${STEPS:-1000} --warmup 20 --no-cpu-baseline >> gpurun_out/bench_$TAG.jsonl 2>> gpurun_out/bench_$TAG.err
done
python tools/show_bench.py gpurun_out/bench_$TAG.jsonl
