# grouped launch order (MRLBM_RAST) with the rotated scalar kernel: C5w / C3
bash tools/ab_libs.sh ab14 "cur cur:MRLBM_RAST=2 cur:MRLBM_RAST=4 cur:MRLBM_RAST=8" "C5 fp64" "C3 fp64"
NO_LAUNCHES=1 MRLBM_RAST=4 bash tools/ncu_capture.sh r03r4 "C5 fp64"
