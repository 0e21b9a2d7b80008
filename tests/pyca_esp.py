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


# --- ESP inbound, independent of oracle/ ---------------------
# Status codes of the readings in DESIGN.md (B1..B9).
OK, DROP_SA, DROP_FORMAT, DROP_REPLAY, DROP_AUTH, DROP_TRAILER = range(6)


class SetWindow:
    """RFC 4303 §3.4.3 receive window kept as the explicit SET of accepted
    numbers plus "everything <= seq0 was received" (reading B6); no bitmap,
    no shifting -- a different construction from the oracle's."""

    def __init__(self, seq0):
        self.top = int(seq0)
        self.seq0 = int(seq0)
        self.seen = set()

    def ok(self, q):
        if q == 0:
            return False
        if q > self.top:
            return True
        if self.top - q >= 64:
            return False
        return not (q <= self.seq0 or q in self.seen)

    def accept(self, q):
        self.seen.add(q)
        self.top = max(self.top, q)

    def bitmap(self):
        """Bits for numbers >= 1 only (bit d <-> number top - d)."""
        b = 0
        for d in range(64):
            x = self.top - d
            if x >= 1 and (x <= self.seq0 or x in self.seen):
                b |= 1 << d
        return b


def encap_raw(spi, key, nonce, hkey, src, dst, q, T, iv=None, tos=0):
    """Outbound with an explicit trailer-included plaintext T (for malformed /
    long-padding test packets)."""
    iv = struct.pack("!Q", q) if iv is None else bytes(iv)
    E = ctr(key, nonce, iv, T)
    H = struct.pack("!II", spi, q) + iv
    icv = hmac.new(bytes(hkey), H + E, hashlib.sha1).digest()[:12]
    tot = 48 + len(T)
    O = struct.pack("!BBHHHBBHII", 0x45, tos, tot, 0, 0x4000, 64, 50, 0, src, dst)
    O = O[:10] + struct.pack("!H", csum(O)) + O[12:]
    return O + H + E + icv


def inbound_one(spi, key, nonce, hkey, win, pkt):
    """(status, inner) for one packet, RFC 4303 §3.4 order."""
    pkt = bytes(pkt)
    L = len(pkt)
    if L < 72 or L > 1552 or (L - 48) % 4:
        return DROP_FORMAT, b""
    if pkt[0] != 0x45 or pkt[9] != 50 or struct.unpack("!H", pkt[2:4])[0] != L:
        return DROP_FORMAT, b""
    if struct.unpack("!H", pkt[6:8])[0] & 0x3FFF or csum(pkt[:20]) != 0:
        return DROP_FORMAT, b""
    if struct.unpack("!I", pkt[20:24])[0] != spi:
        return DROP_FORMAT, b""
    q = struct.unpack("!I", pkt[24:28])[0]
    if not win.ok(q):
        return DROP_REPLAY, b""
    mac = hmac.new(bytes(hkey), pkt[20:L - 12], hashlib.sha1).digest()[:12]
    if not hmac.compare_digest(mac, pkt[L - 12:]):
        return DROP_AUTH, b""
    win.accept(q)
    T = ctr(key, nonce, pkt[28:36], pkt[36:L - 12])
    p = T[-2]
    C = len(T)
    if T[-1] != 4 or p + 22 > C or T[C - 2 - p:C - 2] != bytes(range(1, p + 1)):
        return DROP_TRAILER, b""
    return OK, T[:C - 2 - p]
