# A/B/n: alternate builds of libmrlbm on the same box, 2 reps each.
# usage: LIBS="A=ab/libmrlbm_A.so B=" bash tools/abn.sh TAG "CFG PREC" ...   ("B=" = the in-tree build; env STEPS)
TAG=$1; shift
mkdir -p gpurun_out
for cfg in "$@"; do set -- $cfg
  for rep in 1 2; do
    for lv in ${LIBS:-A=ab/libmrlbm_A.so B=}; do
      name=${lv%%=*}; path=${lv#*=}
      if [ -n "$path" ]; then export MRLBM_LIB=$PWD/$path; else unset MRLBM_LIB; fi
      timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-600} --warmup 20 --no-cpu-baseline $EXTRA > /tmp/b.json 2>>gpurun_out/ab_$TAG.err
      echo "$name $(python tools/show_bench.py /tmp/b.json)" >> gpurun_out/ab_$TAG.txt
    done
  done
done
unset MRLBM_LIB
cat gpurun_out/ab_$TAG.txt
