bash tools/ab_libs.sh ab15 "cur cur:MRLBM_RAST=2 cur:MRLBM_RAST=4" "C4 fp32"
NO_LAUNCHES=1 MRLBM_RAST=4 bash tools/ncu_capture.sh r03r4 "C4 fp32"
