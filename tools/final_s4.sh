# round-1 session-4 evidence: A/B vs the session-start build, default bench line, reference arm, ncu of C2
LIBS="A=ab/libmrlbm_A.so B=" STEPS=1000 bash tools/abn.sh fin "C2 fp64" "C3 fp64" "C4 fp32" > /dev/null
timeout 600 python bench.py > gpurun_out/bench_default_s4.json 2> gpurun_out/bench_default_s4.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/bench_reference_s4.json 2> gpurun_out/bench_reference_s4.err
for cfg in "C2 fp32" "C3 fp64" "C4 fp32" "C5 fp64"; do set -- $cfg
  timeout 300 python bench.py --config $1 --precision $2 --steps 1000 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_all_s4.jsonl 2>> gpurun_out/bench_all_s4.err
done
NO_LAUNCHES= bash tools/ncu_capture.sh r01s4f "C2 fp64" "C5 fp64" > /dev/null 2>&1
cat gpurun_out/ab_fin.txt; python tools/show_bench.py gpurun_out/bench_default_s4.json gpurun_out/bench_all_s4.jsonl; head -c 600 gpurun_out/bench_reference_s4.json
