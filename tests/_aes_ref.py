"""Independent textbook AES-128 (FIPS-197) for checking the AES netlist — test code only.
Written separately from workloads/aes.py (S-box by x^254 in GF(2^8), per-byte state)."""


def _mul(a, b):
    p = 0
    for _ in range(8):
        if b & 1:
            p ^= a
        hi = a & 0x80
        a = (a << 1) & 0xFF
        if hi:
            a ^= 0x1B
        b >>= 1
    return p


def _inv(a):
    r = 1
    for _ in range(254):          # a^254 = a^-1 in GF(2^8) (0 -> 0)
        r = _mul(r, a)
    return r if a else 0


def _sbox(a):
    x = _inv(a)
    y = x
    for s in range(1, 5):
        y ^= ((x << s) | (x >> (8 - s))) & 0xFF
    return y ^ 0x63


SBOX = [_sbox(a) for a in range(256)]


def encrypt(key: bytes, pt: bytes) -> bytes:
    rcon = [0x01, 0x02, 0x04, 0x08, 0x10, 0x20, 0x40, 0x80, 0x1B, 0x36]
    w = [list(key[4 * i:4 * i + 4]) for i in range(4)]
    for i in range(4, 44):
        t = list(w[i - 1])
        if i % 4 == 0:
            t = [SBOX[x] for x in t[1:] + t[:1]]
            t[0] ^= rcon[i // 4 - 1]
        w.append([a ^ b for a, b in zip(w[i - 4], t)])
    s = [pt[i] ^ w[i // 4][i % 4] for i in range(16)]           # s[r + 4c] = byte r of word c
    for rnd in range(1, 11):
        s = [SBOX[x] for x in s]
        s = [s[(r + 4 * ((c + r) % 4))] for c in range(4) for r in range(4)]
        s = [s[r + 4 * c] for c in range(4) for r in range(4)]
        if rnd < 10:
            n = []
            for c in range(4):
                a = s[4 * c:4 * c + 4]
                n += [_mul(a[0], 2) ^ _mul(a[1], 3) ^ a[2] ^ a[3],
                      a[0] ^ _mul(a[1], 2) ^ _mul(a[2], 3) ^ a[3],
                      a[0] ^ a[1] ^ _mul(a[2], 2) ^ _mul(a[3], 3),
                      _mul(a[0], 3) ^ a[1] ^ a[2] ^ _mul(a[3], 2)]
            s = n
        s = [s[i] ^ w[4 * rnd + i // 4][i % 4] for i in range(16)]
    return bytes(s)
