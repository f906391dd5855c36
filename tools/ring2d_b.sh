# 2D TMA ring depth x occupancy x segment, second sweep
TAG=${1:-ring2d_b}
mkdir -p gpurun_out
one() { env $1 timeout 150 python bench.py --config C2 --precision $2 --steps 1000 --no-cpu-baseline --no-e2e | sed "s/^{/{\"lib\": \"$3\", /" >> gpurun_out/${TAG}.jsonl 2>> gpurun_out/${TAG}.err; }
for rep in 1 2; do
  one "MRLBM_TILE=0" fp64 S4m5_seg12; one "MRLBM_TILE=2" fp64 S6m4_seg12; one "MRLBM_TILE=3" fp64 S8m3_seg12
  one "MRLBM_TILE=6" fp64 S5m4_seg12; one "MRLBM_TILE=2 MRLBM_SEG=10" fp64 S6m4_seg10; one "MRLBM_TILE=2 MRLBM_SEG=16" fp64 S6m4_seg16
  one "MRLBM_TILE=4" fp32 S8m5_seg16; one "MRLBM_TILE=7" fp32 S6m6_seg16; one "MRLBM_TILE=4 MRLBM_SEG=20" fp32 S8m5_seg20
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
