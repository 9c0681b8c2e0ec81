"""Host emulation of the degridders' tensor-core operand forms (csrc/idg_kernels_tc.cu: split_fx, split_i8,
the signed-digit limbs of the integer form and its weight classes), with the constants read from the source.

These are bit-level identities of the kernels' arithmetic, checked exhaustively or on large random samples on
the CPU; the GPU parity tests check the kernels' outputs against the oracle.  An fp32 FMA is emulated
exactly: z * sigma (<= 24 + 17 significant bits) + M is exact in fp64, then rounded once to fp32.
"""
import os
import re

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = open(os.path.join(ROOT, "paper_conf_ipps_veenboerpr17_b200", "csrc", "idg_kernels_tc.cu")).read()


def const(name):
    return float(re.search(rf"constexpr float {name} = ([0-9.]+)f;", SRC).group(1))


def prmt(a, b, sel):
    """PTX prmt.b32 (default mode) on uint32 arrays: result byte i = byte (sel >> 4i) & 7 of b:a."""
    src = (b.astype(np.uint64) << np.uint64(32)) | a.astype(np.uint64)
    out = np.zeros_like(a, dtype=np.uint32)
    for i in range(4):
        k = (sel >> (4 * i)) & 7
        byte = (src >> np.uint64(8 * k)) & np.uint64(255)
        out |= (byte.astype(np.uint32) << np.uint32(8 * i))
    return out


def fma32(z, s, m):
    return (z.astype(np.float64) * s + m).astype(np.float32)


def f16_halves(r):
    lo = (r & np.uint32(0xFFFF)).astype(np.uint16).view(np.float16).astype(np.float64)
    hi = (r >> np.uint32(16)).astype(np.uint16).view(np.float16).astype(np.float64)
    return lo, hi


def sample_z(n, seed):
    rng = np.random.default_rng(seed)
    z = rng.uniform(-1.0, 1.0, n).astype(np.float32)
    z[:6] = [1.0, -1.0, 0.0, np.float32(2.0 ** -30), np.float32(0.5), np.float32(-0.999999)]
    return z


def test_fixed_point_f16_split():
    """split_fx: hi + lo = kFxOffset + kFxGain z_q exactly, |z - z_q| <= 0.5 / sigma, both exact f16 values."""
    sigma, magic = const("kFxSigma"), const("kFxMagic")
    offset, gain = const("kFxOffset"), const("kFxGain")
    assert sigma / 128 == gain and magic == 2 ** 23 + 0x680000 + 2 ** 17
    zc, zs = sample_z(1 << 20, 1), sample_z(1 << 20, 2)[::-1].copy()
    wc, ws = fma32(zc, sigma, magic).view(np.uint32), fma32(zs, sigma, magic).view(np.uint32)
    hi, lo = prmt(wc, ws, 0x6521), prmt(wc, ws, 0x7430)
    hc, hs = f16_halves(hi)
    lc, ls = f16_halves(lo)
    for h, l, z in ((hc, lc, zc), (hs, ls, zs)):
        x = np.rint(z.astype(np.float64) * sigma) + 2 ** 17            # X = 2^17 + rn(sigma z)
        assert np.all((h >= 2048) & (h < 4096) & (l >= 14) & (l < 16))
        np.testing.assert_array_equal(h + l, 2062 + x / 128)
        zq = (h + l - offset) / gain
        assert np.max(np.abs(zq - z)) <= 0.5 / sigma * (1 + 1e-6)


def test_integer_split_limbs():
    """split_i8: bytes 0, 1 of fl(sigma z + 2^23 + 2^15) are X = 2^15 + rn(sigma z) (u8 limbs a_l, a_h)."""
    sigma, magic = const("kI8Sigma"), const("kI8Magic")
    assert magic == 2 ** 23 + 2 ** 15
    zc, zs = sample_z(1 << 20, 3), sample_z(1 << 20, 4)
    wc, ws = fma32(zc, sigma, magic).view(np.uint32), fma32(zs, sigma, magic).view(np.uint32)
    a = prmt(wc, ws, 0x5410)                       # (c_l, c_h, s_l, s_h)
    xc = (a & np.uint32(0xFFFF)).astype(np.int64)
    xs = (a >> np.uint32(16)).astype(np.int64)
    np.testing.assert_array_equal(xc, 32768 + np.rint(zc.astype(np.float64) * sigma).astype(np.int64))
    np.testing.assert_array_equal(xs, 32768 + np.rint(zs.astype(np.float64) * sigma).astype(np.int64))
    assert xc.min() >= 1 and xc.max() <= 65535


def signed_digits(x):
    """The kernel's limbs (degridder_setup_tc, BM = 1): x = 2^16 h + 2^8 m + l, each in [-128, 127]."""
    l = ((x + 128) & 255) - 128
    y = (x - l) >> 8
    m = ((y + 128) & 255) - 128
    h = (y - m) >> 8
    return h, m, l


def test_signed_digit_limbs_and_weight_classes():
    rng = np.random.default_rng(5)
    x = rng.integers(-(2 ** 22), 2 ** 22, 1 << 20)
    x[:4] = [2 ** 22 - 1, -(2 ** 22), 0, -1]
    h, m, l = signed_digits(x)
    np.testing.assert_array_equal(65536 * h + 256 * m + l, x)
    for d in (h, m, l):
        assert d.min() >= -128 and d.max() <= 127
    # the three s32 weight classes of one K byte pair (a_l, a_h) against the B bytes (0, h), (h, m), (m, l)
    a_l = rng.integers(0, 256, x.size)
    a_h = rng.integers(0, 256, x.size)
    classes = (2 ** 24) * (a_h * h) + (2 ** 16) * (a_l * h + a_h * m) + (2 ** 8) * (a_l * m + a_h * l)
    np.testing.assert_array_equal(classes, (256 * a_h + a_l) * x - a_l * l)


def test_high_limb_register_is_a_byte_permutation():
    """i8_high_limbs: the (0, x_h) class register from the (x_h, x_m) one by prmt(w16, 0, 0x2404)."""
    rng = np.random.default_rng(6)
    w16 = rng.integers(0, 2 ** 32, 4096, dtype=np.uint64).astype(np.uint32)
    got = prmt(w16, np.zeros_like(w16), 0x2404)
    b = [(w16 >> np.uint32(8 * i)) & np.uint32(255) for i in range(4)]
    np.testing.assert_array_equal(got, (b[0] << np.uint32(8)) | (b[2] << np.uint32(24)))
    assert "0x2404" in SRC and "prmt.b32 %0, %1, 0, 0x2404" in SRC
