# paired kernel fp32: 3-deep (default) vs 5-deep TMA ring (tile 16)
bash tools/ab_libs.sh ab13 "cur cur:MRLBM_TILE=16" "C4 fp32" "C3 fp32" "C5 fp32"
