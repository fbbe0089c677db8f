"""The identity k_svr_udig / k_svr_vdig use to write the SVR operands' balanced base-256 digits
(kernels_svr_tc.cuh, tc_store_digits): for an integer X with |X| <= 2^54, the signed bytes 6..0 of
(X + C) xor C, C = 0x0080808080808080, are the unique digits d_p in [-128, 127] with
X = sum_p d_p 256^(6 - p) -- the digits of the recurrence d = ((X + 128) mod 256) - 128,
X <- (X - d) / 256.  (Host-side check of the arithmetic; the GPU SVR tests compare the path that
uses it with the oracle.)"""
import random

C = 0x0080808080808080


def recurrence(x):
    ds = []
    for _ in range(7):
        d = ((x + 128) & 255) - 128
        x = (x - d) >> 8
        ds.append(d)
    assert x == 0
    return ds[::-1]                                   # most significant first


def bytes_of_xor(x):
    z = ((x + C) & (2 ** 64 - 1)) ^ C
    out = []
    for p in range(7):
        b = (z >> (8 * (6 - p))) & 255
        out.append(b - 256 if b >= 128 else b)
    return out


def test_balanced_digits_identity():
    rng = random.Random(20231112)
    edge = [0, 1, -1, 127, 128, -128, -129, 255, 256, -256, 2 ** 54, -(2 ** 54), 2 ** 54 - 1,
            -(2 ** 54) + 1, 0x7f7f7f7f7f7f, -0x7f7f7f7f7f7f]
    xs = edge + [rng.randint(-(2 ** 54), 2 ** 54) for _ in range(50000)] + \
        [rng.choice((-1, 1)) * rng.randint(0, 2 ** rng.randint(0, 54)) for _ in range(50000)]
    for x in xs:
        d = bytes_of_xor(x)
        assert d == recurrence(x), x
        assert all(-128 <= v <= 127 for v in d)
        assert sum(v * 256 ** (6 - p) for p, v in enumerate(d)) == x
