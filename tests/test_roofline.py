"""Pins of the performance-model arithmetic to the paper's Tables 2-3 and the
P:L310 memory numbers (exact arithmetic from Table 1 bandwidths)."""
import pytest

from paper_conf_sc_valero_laravgr23_b200 import roofline


def test_table2_bytes_per_flup():
    # Table 2, P:L295-300 (double precision)
    assert roofline.bytes_per_lup("D2Q9", "ST") == 144
    assert roofline.bytes_per_lup("D3Q19", "ST") == 304
    assert roofline.bytes_per_lup("D2Q9", "MR") == 96
    assert roofline.bytes_per_lup("D3Q19", "MR") == 160


@pytest.mark.parametrize("bw,lat,pat,expect", [
    (900e9, "D2Q9", "ST", 6250), (900e9, "D3Q19", "ST", 2960), (900e9, "D2Q9", "MR", 9375),
    (900e9, "D3Q19", "MR", 5625), (1228.86e9, "D2Q9", "ST", 8533), (1228.86e9, "D3Q19", "ST", 4042),
    (1228.86e9, "D2Q9", "MR", 12800), (1228.86e9, "D3Q19", "MR", 7680)])
def test_table3_roofline(bw, lat, pat, expect):
    # Table 3, from Table 1 bandwidths and eq 15
    assert int(roofline.mflups_max(bw, lat, pat)) == expect


def test_memory_claims_p310():
    gib = 2 ** 30
    assert round(roofline.memory_bytes(15_000_000, "D2Q9", "MR") / gib, 2) == 1.34   # "1.3GB"
    assert round(roofline.memory_bytes(15_000_000, "D3Q19", "MR") / gib, 2) == 2.24  # "2.23GB"
    assert round(roofline.memory_bytes(15_000_000, "D2Q9", "ST") / gib, 1) == 2.0    # "about 2GB"
    assert round(roofline.memory_bytes(15_000_000, "D3Q19", "ST") / gib, 1) == 4.2   # "4.2GB"
    # the reductions of the abstract: ~35% and ~47%
    r2 = 1 - roofline.memory_bytes(1, "D2Q9", "MR") / roofline.memory_bytes(1, "D2Q9", "ST")
    r3 = 1 - roofline.memory_bytes(1, "D3Q19", "MR") / roofline.memory_bytes(1, "D3Q19", "ST")
    assert round(r2, 2) == 0.33 and round(r3, 2) == 0.47
