# numerical A/B of the D3Q27-R formulations (fp32, 1000 steps): product form (in-tree) vs collide + synthesis (q0)
for bc in periodic cavity open_x; do
  timeout 600 python tools/parity_probe.py D3Q27 recursive $bc fp32 2>&1 | tail -1 | sed 's/^/product /'
  MRLBM_LIB=$PWD/ab/libmrlbm_q0.so timeout 600 python tools/parity_probe.py D3Q27 recursive $bc fp32 2>&1 | tail -1 | sed 's/^/q0      /'
  MRLBM_TILE=9 timeout 600 python tools/parity_probe.py D3Q27 recursive $bc fp32 2>&1 | tail -1 | sed 's/^/oldkern /'
done
