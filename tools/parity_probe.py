"""Print the per-group parity errors of one long-parity case for the library in
MRLBM_LIB (A/B of numerically different kernel formulations; not a test).
usage: python tools/parity_probe.py LAT REG BC PRECISION [STEPS]"""
import sys
from pathlib import Path

sys.path.insert(0, str(Path(__file__).resolve().parents[1] / "tests"))
sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import test_gpu_parity_long as T  # noqa: E402
from parity import group_errors  # noqa: E402

lat, reg, bc, prec = sys.argv[1:5]
if len(sys.argv) > 5:
    T.STEPS = int(sys.argv[5])


class MP:  # minimal monkeypatch stand-in
    def setenv(self, k, v):
        import os
        os.environ[k] = v

    def delenv(self, k, raising=False):
        import os
        os.environ.pop(k, None)


print(lat, reg, bc, prec, T.STEPS, T.run_gpu(lat, reg, bc, prec, None, MP()))
