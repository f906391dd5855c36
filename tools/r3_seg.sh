# round 3: sanitizer on the new default kernels, then the 3D segment-length sweep with them
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_slabs.py -m gpu -q > gpurun_out/pytest_r03_p2p.log 2>&1; tail -n 3 gpurun_out/pytest_r03_p2p.log
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  for c in 3d p2p; do
    timeout 1200 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_case.py $c > gpurun_out/sanitize_r03_${tool}_${c}.log 2>&1
    echo "$tool $c rc=$? $(grep -c '^ok' gpurun_out/sanitize_r03_${tool}_${c}.log) ok; $(grep -m1 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/sanitize_r03_${tool}_${c}.log)"
  done
done
for cfg in "C3 fp64" "C5 fp64" "C4 fp32"; do set -- $cfg
  for seg in 0 24 48 64 96; do
    MRLBM_SEG=$seg timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline --no-e2e | sed "s/^{/{\"lib\": \"seg$seg\", /" >> gpurun_out/seg_r03.jsonl
  done
done
python tools/show_ab.py gpurun_out/seg_r03.jsonl
