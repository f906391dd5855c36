# A/B: ab/libmrlbm_A.so (baseline) vs the in-tree library, alternating, 2 reps;
# usage: bash tools/ab2.sh TAG "CFG PREC" ...   (env STEPS)
TAG=$1; shift
mkdir -p gpurun_out
for cfg in "$@"; do set -- $cfg
  for rep in 1 2; do
    for v in A B; do
      if [ $v = A ]; then export MRLBM_LIB=$PWD/ab/libmrlbm_A.so; else unset MRLBM_LIB; fi
      timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-600} --warmup 20 --no-cpu-baseline > /tmp/b.json 2>>gpurun_out/ab_$TAG.err
      echo "$v $(python tools/show_bench.py /tmp/b.json)" >> gpurun_out/ab_$TAG.txt
    done
  done
done
unset MRLBM_LIB
cat gpurun_out/ab_$TAG.txt
