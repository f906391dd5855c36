# usage: bash tools/sweep.sh TAG "CFG PREC" ...  (env grid: TILES, SEGS)
TAG=$1; shift
for cfg in "$@"; do set -- $cfg
  for t in ${TILES:-0}; do for sg in ${SEGS:-0}; do
    MRLBM_TILE=$t MRLBM_SEG=$sg timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-600} --warmup 20 --no-cpu-baseline > /tmp/b.json 2>>gpurun_out/sweep_$TAG.err
    echo "tile=$t seg=$sg $(python tools/show_bench.py /tmp/b.json)" >> gpurun_out/sweep_$TAG.txt
  done; done
done
cat gpurun_out/sweep_$TAG.txt
