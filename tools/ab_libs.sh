# one-box A/B of library builds: bash tools/ab_libs.sh TAG "lib1 lib2 ..." "CFG PREC" ...
# libN = ab/libmrlbm_N.so ("cur" = the in-tree build), optionally "name:VAR=val" (env for that arm); runs GPU tests first when PYTEST=1
TAG=$1; LIBS=$2; shift 2
CFGS=("$@")
mkdir -p gpurun_out
if [ -n "$PYTEST" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/${TAG}_pytest.log 2>&1; tail -2 gpurun_out/${TAG}_pytest.log
fi
for rep in 1 2; do
for cfg in "${CFGS[@]}"; do set -- $cfg
  for lib in $LIBS; do
    name=${lib%%:*}; envs=""; [ "$name" != "$lib" ] && envs=${lib#*:}
    if [ "$name" = cur ]; then L=""; else L=$PWD/ab/libmrlbm_$name.so; fi
    env $envs MRLBM_LIB=$L timeout 300 python bench.py --config $1 --precision $2 --steps ${STEPS:-200} --no-cpu-baseline --no-e2e $EXTRA | sed "s/^{/{\"lib\": \"$lib\", /" >> gpurun_out/${TAG}.jsonl
  done
done
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
