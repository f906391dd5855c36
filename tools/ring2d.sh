# 2D TMA ring depth for fp32 (MRLBM_TILE 0: S=4, 4: S=8, 5: S=12; all 5 CTAs/SM min) x segment length
TAG=${1:-ring2d}
mkdir -p gpurun_out
one() { env $1 timeout 150 python bench.py --config C2 --precision $2 --steps 1000 --no-cpu-baseline --no-e2e | sed "s/^{/{\"lib\": \"$3\", /" >> gpurun_out/${TAG}.jsonl 2>> gpurun_out/${TAG}.err; }
for rep in 1 2; do
  one "MRLBM_TILE=0" fp32 S4_seg16; one "MRLBM_TILE=4" fp32 S8_seg16; one "MRLBM_TILE=5" fp32 S12_seg16
  one "MRLBM_TILE=4 MRLBM_SEG=12" fp32 S8_seg12; one "MRLBM_TILE=4 MRLBM_SEG=24" fp32 S8_seg24
  one "MRLBM_TILE=0" fp64 S4_seg12; one "MRLBM_TILE=2" fp64 S6_seg12_4cta
done
python tools/show_ab.py gpurun_out/${TAG}.jsonl
