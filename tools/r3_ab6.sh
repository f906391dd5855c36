# p6 (paired kernel, old kernel with the regrouped D3Q19 collision): one-box A/B + ncu of the C3/C5 candidates
bash tools/ab_libs.sh ab6 "base cur cur:MRLBM_TILE=9 cur:MRLBM_TILE=10 cur:MRLBM_TILE=11" "C4 fp32" "C5 fp64" "C3 fp64"
NO_LAUNCHES=1 MRLBM_TILE=9 bash tools/ncu_capture.sh r03c_t9 "C3 fp64" "C5 fp64"
NO_LAUNCHES=1 MRLBM_TILE=11 bash tools/ncu_capture.sh r03c_t11 "C3 fp64" "C5 fp64"
NO_LAUNCHES=1 bash tools/ncu_capture.sh r03c_t0 "C3 fp64"
