# p11: regrouped D3Q27-R collision (fp32 paired kernel): precision probe + A/B + D3Q27 parity
for bc in periodic cavity open_x; do
  timeout 600 python tools/parity_probe.py D3Q27 recursive $bc fp32 2>&1 | tail -1 | sed 's/^/p11 /'
done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_long.py tests/test_gpu_fullsize.py -m gpu -q -x -k "D3Q27 or C4" > gpurun_out/ab9_pytest.log 2>&1; tail -n 2 gpurun_out/ab9_pytest.log
bash tools/ab_libs.sh ab9 "p10 cur" "C4 fp32" "C4 fp64"
