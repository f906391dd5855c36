# compute-sanitizer memcheck / racecheck / synccheck on small cases of the fused step
# (tools/sanitize_case.py); logs under gpurun_out/sanitize_<tool>_<case>.log
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  for c in 2d 3d p2p; do
    timeout 900 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_case.py $c \
      > gpurun_out/sanitize_${tool}_${c}.log 2>&1
    echo "$tool $c rc=$? $(grep -c '^ok' gpurun_out/sanitize_${tool}_${c}.log) ok; $(grep -m1 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_${c}.log)"
  done
  MRLBM_CLUSTER=2 timeout 900 $CS --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_case.py 3d \
    > gpurun_out/sanitize_${tool}_3d_cluster.log 2>&1
  echo "$tool 3d cluster rc=$? $(grep -m1 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_3d_cluster.log)"
done
