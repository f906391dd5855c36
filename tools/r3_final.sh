# round-3 evidence on one box: GPU suite, smoke, default bench line, every config (MR + ST),
# the reference arm, ncu --set full of each workload's step kernel, launch list of the default line
TAG=${1:-r03}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > gpurun_out/smi_$TAG.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/pytest_$TAG.log 2>&1; tail -n 2 gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -n 1 gpurun_out/smoke_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_${TAG}_default.json 2> gpurun_out/bench_${TAG}_default.err; tail -c 300 gpurun_out/bench_${TAG}_default.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_${TAG}_reference.json 2> gpurun_out/bench_${TAG}_reference.err; tail -c 200 gpurun_out/bench_${TAG}_reference.json
for cfg in "C2 fp32 MR" "C3 fp64 MR" "C3 fp32 MR" "C4 fp32 MR" "C5 fp64 MR" "C5 fp32 MR" "C1 fp64 MR" "C2 fp64 ST" "C3 fp64 ST" "C4 fp32 ST"; do set -- $cfg
  timeout 400 python bench.py --config $1 --precision $2 --method $3 --steps ${STEPS:-200} --no-cpu-baseline >> gpurun_out/bench_${TAG}_all.jsonl 2>> gpurun_out/bench_${TAG}_all.err
done
python tools/show_bench.py gpurun_out/bench_${TAG}_all.jsonl
NO_LAUNCHES= bash tools/ncu_capture.sh $TAG "C2 fp64" "C2 fp32" "C3 fp64" "C4 fp32" "C5 fp64"
