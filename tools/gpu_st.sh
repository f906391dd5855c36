# ST tests + MR-vs-ST bench lines + ncu captures (C3 MR, C3 ST); usage: bash tools/gpu_st.sh TAG
TAG=$1
timeout 900 python -m pytest tests/test_gpu_st.py -q -x --timeout 600 > gpurun_out/pytest_st_$TAG.log 2>&1; tail -3 gpurun_out/pytest_st_$TAG.log
for cfg in "C2 fp64 MR" "C2 fp64 ST" "C2 fp32 ST" "C3 fp64 MR" "C3 fp64 ST" "C4 fp32 ST"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --method $3 --steps ${STEPS:-500} --warmup 20 --no-cpu-baseline >> gpurun_out/bench_st_$TAG.jsonl 2>> gpurun_out/bench_st_$TAG.err
done
python tools/show_bench.py gpurun_out/bench_st_$TAG.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mrlbm_step -s 5 -c 1 -o gpurun_out/ncu_C3_MR_$TAG python bench.py --config C3 --steps 8 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:st_step -s 5 -c 1 -o gpurun_out/ncu_C3_ST_$TAG python bench.py --config C3 --method ST --steps 8 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ls gpurun_out
