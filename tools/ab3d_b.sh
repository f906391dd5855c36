# A/B round 2b: new default vs ROT3 (D3Q27-R) vs no-barrier timing bound vs 32x8 tile for C4
TAG=${1:-ab}
mkdir -p gpurun_out
run() { # lib-tag env... -- bench args
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 200 --no-cpu-baseline $BARGS | sed "s/^{/{\"lib\": \"$tag\", /" >> gpurun_out/${TAG}.jsonl
}
for rep in 1 2; do
  BARGS="--config C4 --precision fp32"
  run new X=1; run rot3 MRLBM_LIB=$PWD/ab/libmrlbm_rot3.so; run nobar MRLBM_LIB=$PWD/ab/libmrlbm_nobar.so; run tile1 MRLBM_TILE=1
  BARGS="--config C5 --precision fp64"
  run new X=1; run nobar MRLBM_LIB=$PWD/ab/libmrlbm_nobar.so
  BARGS="--config C3 --precision fp64"
  run new X=1; run nobar MRLBM_LIB=$PWD/ab/libmrlbm_nobar.so
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
