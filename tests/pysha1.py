"""Tiny pure-Python SHA-1 compression (FIPS 180-4 §6.1.2), tests only.

Used to continue from the library's exported HMAC midstates, so that the
midstate precomputation can be pinned to RFC 2202 digests without a GPU."""
import struct


def _rol(x, n):
    return ((x << n) | (x >> (32 - n))) & 0xFFFFFFFF


def compress(h, block):
    w = list(struct.unpack(">16I", block))
    for t in range(16, 80):
        w.append(_rol(w[t - 3] ^ w[t - 8] ^ w[t - 14] ^ w[t - 16], 1))
    a, b, c, d, e = h
    for t in range(80):
        if t < 20:
            f, k = (b & c) | (~b & d), 0x5A827999
        elif t < 40:
            f, k = b ^ c ^ d, 0x6ED9EBA1
        elif t < 60:
            f, k = (b & c) | (b & d) | (c & d), 0x8F1BBCDC
        else:
            f, k = b ^ c ^ d, 0xCA62C1D6
        a, b, c, d, e = (_rol(a, 5) + f + e + k + w[t]) & 0xFFFFFFFF, a, _rol(b, 30), c, d
    return [(x + y) & 0xFFFFFFFF for x, y in zip(h, (a, b, c, d, e))]


def finish(h, msg, prefix_len):
    """SHA-1 of (prefix || msg) given the state h after the prefix blocks."""
    total = prefix_len + len(msg)
    m = msg + b"\x80" + b"\x00" * ((55 - total) % 64) + struct.pack(">Q", total * 8)
    for i in range(0, len(m), 64):
        h = compress(h, m[i:i + 64])
    return struct.pack(">5I", *h)
