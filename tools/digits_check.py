"""Exhaustive host check of the kernels' norm-digit builder (tid_kernels.cu norm_digits): the byte-permute rank
words equal the greedy encoding of E = floor(W / 2) for every column term W in [0, 2^21].  python tools/digits_check.py"""
import numpy as np
W = np.arange(0, 2**21 + 1, dtype=np.int64)   # max W = 128*128*128 = 2,097,152 (sum r(256-r) over 128 bytes)
E = W >> 1
hi = E // 255; lo = E - 255 * hi
q = hi // 255; rem = hi - 255 * q
# reference: greedy digit of rank k = clamp(hi - 255 k, 0, 255), ranks 0..29
ranks = np.clip(hi[:, None] - 255 * np.arange(30)[None, :], 0, 255)
ref = np.zeros((len(W), 32), np.int64)
pos = list(range(15)) + list(range(16, 31))
ref[:, pos] = ranks
ref[:, 15] = lo
# new builder: rank words via byte_perm(0, b, sel)
Wc = 0x0000000455555555
b = 0xFFFFFF00 | rem
rk = np.zeros((len(W), 8), np.int64)
for i in range(8):
    s = np.clip(32 - 4 * q + 16 * i, 12, 36)
    sel = (Wc >> s) & 0xFFFF
    word = np.zeros(len(W), np.int64)
    for p in range(4):
        nib = (sel >> (4 * p)) & 7
        src = np.where(nib < 4, 0, (b >> (8 * (nib - 4))) & 0xFF)
        word |= src << (8 * p)
    rk[:, i] = word
def bp(x, y, s):  # __byte_perm(x, y, s) without sign mode
    out = np.zeros_like(x)
    for p in range(4):
        nib = (s >> (4 * p)) & 7
        val = np.where(nib < 4, (x >> (8 * (nib % 4))) & 0xFF, (y >> (8 * (nib - 4))) & 0xFF)
        out |= val << (8 * p)
    return out
w8 = np.zeros((len(W), 8), np.int64)
w8[:, 0] = rk[:, 0]; w8[:, 1] = rk[:, 1]; w8[:, 2] = rk[:, 2]
w8[:, 3] = (rk[:, 3] & 0x00FFFFFF) | (lo << 24)
w8[:, 4] = bp(rk[:, 3], rk[:, 4], 0x6543)
w8[:, 5] = bp(rk[:, 4], rk[:, 5], 0x6543)
w8[:, 6] = bp(rk[:, 5], rk[:, 6], 0x6543)
w8[:, 7] = bp(rk[:, 6], rk[:, 7], 0x6543) & 0x00FFFFFF
got = np.zeros((len(W), 32), np.int64)
for i in range(8):
    for p in range(4):
        got[:, 4 * i + p] = (w8[:, i] >> (8 * p)) & 0xFF
assert (got == ref).all(), np.argwhere(got != ref)[:5]
# and the digits reproduce E against the constant operand (255 x 15, 1, 255 x 15, 1)
a = np.array([255] * 15 + [1] + [255] * 15 + [1])
assert ((got * a).sum(1) == E).all()
print("byte-permute rank builder == greedy digits for every W in [0, 2^21]")
