# p10: per-lattice defaults (D3Q19 scalar kernel + regrouped collision, D3Q27 paired 32x8; D3Q27-R fp64 product form)
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/ab8_pytest.log 2>&1; tail -n 2 gpurun_out/ab8_pytest.log
bash tools/ab_libs.sh ab8 "base cur cur:MRLBM_TILE=9 cur:MRLBM_TILE=10" "C3 fp64" "C5 fp64" "C4 fp32" "C3 fp32" "C5 fp32" "C4 fp64"
