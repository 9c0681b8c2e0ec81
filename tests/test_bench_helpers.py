"""bench.py host helpers (no GPU): sincos-per-pair accounting of each kernel family and the
one-line JSON contract of the reference arm's shape."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_sincos_per_pair_by_family():
    spp = bench.sincos_per_pair
    assert spp("gridder_tc<24,W12,MT3,minB2>", 16) == 1.0          # the paper's one sincos per pair
    assert spp("degridder_tc<24,W8,MT2,minB4>", 16) == 1.0
    assert spp("gridder_rot2<24,W12,MT3,minB2,KPT2>", 16) == 0.5     # group-0 phasors only
    assert spp("gridder_rot2<32,W16,MT4,minB2,KPT4,GP2>", 32) == 0.25
    assert spp("gridder_rot<24,W12,MT3,minB2,KPT4>", 16) == 0.75     # + E_t per lane
    assert spp("degridder_rot<24,W8,minB4,U1,C16>", 16) == 0.5       # row 0 + E for 4 rows
    assert spp("degridder_rot8<24,W8,minB2,U1,C16>", 16) == 0.25
    assert spp("degridder_rot16<24,W4,minB3,U4,C16>", 16) == 0.125
    assert spp("degridder_rot16s2<32,W8,minB2,U2,C32>", 32) == 0.1875  # + row 8 (second chain)


def test_ops_per_pair_is_the_papers():
    # 17 FMA + 1 sincos = 36 paper-ops per (pixel, visibility) pair
    assert bench.OPS_PER_PAIR == 36


def test_sincos_fma_roofline_unit_counts():
    # 148 SMs x min(128/17, 16/2) pairs/clk x 36 ops at 1965 MHz = 78.8 TOps/s
    assert abs(bench.sincos_fma_roofline(1965) - 78.84) < 0.05


def test_step_kind_per_config():
    assert bench.STEP_KIND["predict"] == "degrid"                  # configs[4]: degridding-only sweep
    assert all(bench.STEP_KIND[c] == "grid+degrid" for c in ("tiny", "lofar", "lofar_dde", "ska"))
    assert bench.E2E_TIME_CHUNK["ska"] == 1024                      # 8 chunks of 1024


def test_tensor_ops_per_pair():
    from bench import tensor_ops_per_pair as top
    assert top("degridder_rot16i<32,W4,minB2,U4,C32>")[0] == 192    # integer form: 3 classes x 32 MACs x 2
    assert top("degridder_rot16<24,W4,minB3,U4,C16>")[0] == 96      # f16 fixed-point split: 3 x 16 x 2
    for name in ("degridder_roti<24,W8,minB3,U1,C4>", "degridder_rot8i<24,W4,minB3,U2,C16>", "degridder_tci<32,W8,MT2,minB2>"):
        assert top(name)[0] == 192, name
    assert top("degridder_tc<32,W8,MT4,minB2>")[0] == 96
    assert top("gridder_rot2h<32,W16,MT4,minB2,KPT4,GP4,lmnsm>")[0] == 96
