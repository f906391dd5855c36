# round-3 exploration on one box: pipe microbenchmark + existing 3D tile variants (A/B, same box)
# usage: bash tools/r3_explore.sh TAG
TAG=${1:-r3x}
mkdir -p gpurun_out
./tools/ubench_pipes > gpurun_out/${TAG}_ubench.txt 2>&1
for cfg in "C3 fp64 0" "C3 fp64 2" "C5 fp64 0" "C5 fp64 2" "C4 fp32 0" "C4 fp32 3" "C4 fp32 1"; do set -- $cfg
  MRLBM_TILE=$3 timeout 300 python bench.py --config $1 --precision $2 --steps 200 --no-cpu-baseline --no-e2e | sed "s/^{/{\"lib\": \"tile$3\", /" >> gpurun_out/${TAG}.jsonl
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
