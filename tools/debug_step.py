"""Debug helper: run a few steps of one variant and print parity vs the oracle."""
import sys, time
sys.path.insert(0, '.')
sys.path.insert(0, 'tests')
import numpy as np
from paper_conf_sc_valero_laravgr23_b200 import inputs, mrlbm
import oracle
lat = sys.argv[1] if len(sys.argv) > 1 else "D2Q9"
reg = sys.argv[2] if len(sys.argv) > 2 else "projective"
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
prec = sys.argv[4] if len(sys.argv) > 4 else "fp64"
D = 2 if lat == "D2Q9" else 3
nx, ny, nz = (40, 9, 1) if D == 2 else (33, 9, 5)
m0 = inputs.random_state(D, nx, ny, nz, U=0.05) if "rand" in sys.argv else inputs.perturbed_rest(D, nx, ny, nz, U=0.05)
s = mrlbm.Solver(lat, nx, ny, nz, 0.7, reg, {}, precision=prec)
print("config", s.kernel_config(), flush=True)
s.set_moments(m0)
print("set ok", np.abs(s.get_moments() - m0).max(), flush=True)
s.step(steps)
s.sync()
print("step ok", flush=True)
got = s.get_moments()
o = oracle.Oracle(lat, nx, ny, nz, 0.7, reg)
o.set_moments(m0); o.step(steps); ref = o.get_moments()
from parity import group_errors
print(lat, reg, steps, prec, group_errors(got, ref, D), "abs", np.abs(got-ref).max(), flush=True)
