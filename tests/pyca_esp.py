"""Independent third composition of ESP outbound/inbound (tests only).

Built from pyca `cryptography` (OpenSSL AES-CTR) and the Python stdlib
`hmac`/`hashlib` (OpenSSL SHA-1), following the same readings A1..A17
(DESIGN.md §3).  It shares no code with oracle/ (plain C) or the CUDA path; it
is one of the pins the oracle is checked against.
"""
import hashlib
import hmac
import struct

from cryptography.hazmat.primitives.ciphers import Cipher, algorithms, modes


def ctr(key, nonce, iv, data):
    icb = bytes(nonce) + bytes(iv) + b"\x00\x00\x00\x01"
    e = Cipher(algorithms.AES(bytes(key)), modes.CTR(icb)).encryptor()
    return e.update(bytes(data)) + e.finalize()


def csum(h):
    s = sum(struct.unpack("!%dH" % (len(h) // 2), h))
    while s >> 16:
        s = (s & 0xFFFF) + (s >> 16)
    return (~s) & 0xFFFF


def encap(spi, key, nonce, hkey, src, dst, q, P):
    P = bytes(P)
    D = len(P)
    p = (-(D + 2)) % 4
    T = P + bytes(range(1, p + 1)) + bytes([p, 4])
    iv = struct.pack("!Q", q)
    E = ctr(key, nonce, iv, T)
    H = struct.pack("!II", spi, q) + iv
    icv = hmac.new(bytes(hkey), H + E, hashlib.sha1).digest()[:12]
    tot = 48 + len(T)
    O = struct.pack("!BBHHHBBHII", 0x45, P[1], tot, 0, 0x4000, 64, 50, 0, src, dst)
    O = O[:10] + struct.pack("!H", csum(O)) + O[12:]
    return O + H + E + icv


def decap(key, nonce, hkey, pkt):
    pkt = bytes(pkt)
    assert csum(pkt[:20]) == 0
    H, rest = pkt[20:36], pkt[36:]
    E, icv = rest[:-12], rest[-12:]
    assert hmac.compare_digest(hmac.new(bytes(hkey), H + E, hashlib.sha1).digest()[:12], icv)
    T = ctr(key, nonce, H[8:16], E)
    p = T[-2]
    assert T[-1] == 4 and p <= 3
    assert T[len(T) - 2 - p:len(T) - 2] == bytes(range(1, p + 1))
    return T[:len(T) - 2 - p], struct.unpack("!I", H[4:8])[0]
