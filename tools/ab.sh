# A/B: ab/libmrlbm_A.so (baseline) vs the in-tree library, alternating; usage: bash tools/ab.sh TAG "CFG PREC" ...
TAG=$1; shift
for cfg in "$@"; do set -- $cfg
  for rep in 1 2; do
    for v in A B; do
      if [ $v = A ]; then export MRLBM_LIB=$PWD/ab/libmrlbm_A.so; else unset MRLBM_LIB; fi
      timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-1000} --warmup 20 --no-cpu-baseline > /tmp/b.json 2>>gpurun_out/ab_$TAG.err
      echo "$v $(python tools/show_bench.py /tmp/b.json)" >> gpurun_out/ab_$TAG.txt
    done
  done
done
unset MRLBM_LIB
cat gpurun_out/ab_$TAG.txt
