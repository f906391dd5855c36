# round-1 session-5: validate the boundary-free-interior build (GPU tests, smoke, bench lines, ncu)
bash tools/gpu_check.sh s5
timeout 600 python bench.py > gpurun_out/bench_default_s5.json 2> gpurun_out/bench_default_s5.err
timeout 600 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/bench_reference_s5.json 2> gpurun_out/bench_reference_s5.err
timeout 300 python bench.py --config C5 --precision fp64 --steps 1000 --warmup 20 --no-cpu-baseline >> gpurun_out/bench_s5.jsonl 2>> gpurun_out/bench_s5.err
NO_LAUNCHES= bash tools/ncu_capture.sh r01s5 "C2 fp64" "C5 fp64" > /dev/null 2>&1
python tools/show_bench.py gpurun_out/bench_default_s5.json; head -c 600 gpurun_out/bench_reference_s5.json
