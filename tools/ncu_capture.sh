# usage: bash tools/ncu_capture.sh TAG "CFG PREC" ...  -- one ncu --set full capture of the fused
# step kernel per workload, exported on the box (raw + source pages as CSV; the .ncu-rep is kept
# only when small, gpurun copies back at most 64 MiB) + the C2 launch list
TAG=$1; shift
mkdir -p gpurun_out
for cfg in "$@"; do set -- $cfg
  R=gpurun_out/prof_${TAG}_$1_$2
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:mrlbm_step -s 5 -c 1 \
    -o /tmp/prof_${TAG}_$1_$2 -f python bench.py --config $1 --precision $2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e \
    > ${R}.log 2>&1; tail -1 ${R}.log
  ncu -i /tmp/prof_${TAG}_$1_$2.ncu-rep --page raw --csv > ${R}_raw.csv 2>/dev/null
  ncu -i /tmp/prof_${TAG}_$1_$2.ncu-rep --page source --csv --print-source sass > ${R}_sass.csv 2>/dev/null
  ncu -i /tmp/prof_${TAG}_$1_$2.ncu-rep --page details > ${R}_details.txt 2>/dev/null
  gzip -f ${R}_sass.csv
  sz=$(stat -c %s /tmp/prof_${TAG}_$1_$2.ncu-rep); [ "$sz" -lt 12000000 ] && cp /tmp/prof_${TAG}_$1_$2.ncu-rep gpurun_out/
done
if [ -z "$NO_LAUNCHES" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_${TAG}_C2.csv \
  python bench.py --steps 300 --warmup 10 --no-cpu-baseline > gpurun_out/launches_${TAG}.log 2>&1; tail -1 gpurun_out/launches_${TAG}.log | cut -c1-200
fi
du -sh gpurun_out
