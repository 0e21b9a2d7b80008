"""Seeded synthetic workload generator (SA tables + packet batches).

This module holds NONE of the method's arithmetic (no AES, SHA-1, HMAC, ESP
framing or outer-header logic).  It only synthesises inputs, and it is the one
piece of code shared by the CUDA path's tests/bench and the oracle.

Workload recipe:
  * "randomly generated IP traffic with UDP payloads", IPv4 headers for IPsec
    (§4.1 "Workloads");
  * packet sizes 64..1514 B frames (Fig. 12(c) x-axis), IMIX
    64/594/1514 at 7:4:1 (BASELINE.json configs[3]);
  * 1024 SAs, random keys (BASELINE.json north_star; per-flow contexts
    PAPER.md:395).
Frame length L excludes the FCS; the library sees only the inner IPv4
datagram, D = L - 14 (reading A2).
"""
from __future__ import annotations

import dataclasses

import numpy as np

SEED = 20150421
SLOT = 2048          # packet-pool slot stride (bytes)
HEADROOM = 128       # headroom before the Ethernet header in each slot
ETH = 14
IMIX_SIZES = (64, 594, 1514)
IMIX_WEIGHTS = (7, 4, 1)
TUN_SRC = (192 << 24) | (0 << 16) | (2 << 8) | 1          # 192.0.2.1 (RFC 5737)
TUN_DST_BASE = (198 << 24) | (51 << 16) | (100 << 8)      # 198.51.100.0/24


def rng_for(cfg_id: int, rank: int = 0, batch: int = 0, salt: int = 0) -> np.random.Generator:
    return np.random.default_rng([SEED, cfg_id, rank, batch, salt])


@dataclasses.dataclass
class SAParams:
    """SoA security-association parameters (host order integers)."""
    spi: np.ndarray          # u32[n]
    tunnel_src: np.ndarray   # u32[n]
    tunnel_dst: np.ndarray   # u32[n]
    aes_key: np.ndarray      # u8[n,16]
    ctr_nonce: np.ndarray    # u8[n,4]
    hmac_key: np.ndarray     # u8[n,20]
    seq: np.ndarray          # u32[n]

    def __len__(self):
        return int(self.spi.shape[0])

    def copy(self) -> "SAParams":
        return SAParams(*(np.array(getattr(self, f.name)) for f in dataclasses.fields(self)))


@dataclasses.dataclass
class Batch:
    n: int
    in_buf: np.ndarray       # u8[pool]
    in_off: np.ndarray       # u32[n]  offset of the inner IPv4 datagram
    in_len: np.ndarray       # u16[n]  D
    sa_idx: np.ndarray       # u32[n]
    out_off: np.ndarray      # u32[n]
    out_pool_bytes: int
    frame_len: np.ndarray    # u32[n]  L (for Gbps accounting, reading A18)


def make_sas(n_sa: int, cfg_id: int = 0, rank: int = 0, world: int = 1,
             seq0: int | np.ndarray = 0) -> SAParams:
    """SA table for one rank: global SA ids s = rank + world*j (SA-hash shard)."""
    r = rng_for(cfg_id, rank, 0, salt=1)
    gid = rank + world * np.arange(n_sa, dtype=np.int64)
    seq = np.full(n_sa, 0, np.uint32) if np.isscalar(seq0) else np.asarray(seq0, np.uint32)
    if np.isscalar(seq0):
        seq[:] = np.uint32(seq0)
    return SAParams(
        spi=(0x100 + gid).astype(np.uint32),
        tunnel_src=np.full(n_sa, TUN_SRC, np.uint32),
        tunnel_dst=(TUN_DST_BASE + (gid % 254) + 1).astype(np.uint32),
        aes_key=r.integers(0, 256, (n_sa, 16), dtype=np.uint8),
        ctr_nonce=r.integers(0, 256, (n_sa, 4), dtype=np.uint8),
        hmac_key=r.integers(0, 256, (n_sa, 20), dtype=np.uint8),
        seq=seq,
    )


def frame_sizes(n: int, size, r: np.random.Generator) -> np.ndarray:
    """Frame lengths L for n packets: an int, 'imix', or an explicit array."""
    if isinstance(size, str):
        assert size == "imix"
        w = np.array(IMIX_WEIGHTS, np.int64)
        counts = (n * w) // w.sum()
        for j in range(int(n - counts.sum())):           # leftovers to the largest sizes
            counts[len(w) - 1 - j] += 1                   # (65536 -> 38229/21845/5462)
        L = np.repeat(np.array(IMIX_SIZES, np.uint32), counts)
        return L[r.permutation(n)]                          # Fisher-Yates shuffle
    if np.isscalar(size):
        return np.full(n, int(size), np.uint32)
    a = np.asarray(size, np.uint32)
    assert a.shape == (n,)
    return a


def _csum16(words: np.ndarray) -> np.ndarray:
    """Input synthesis only: inner IPv4 header checksum for realism."""
    s = words.astype(np.uint64).sum(axis=1)
    while np.any(s >> 16):
        s = (s & 0xFFFF) + (s >> 16)
    return (~s & 0xFFFF).astype(np.uint16)


def make_batch(n: int, size, n_sa: int, cfg_id: int = 0, rank: int = 0, batch: int = 0,
               locality: int = 1, layout: str = "slots", in_len_override=None,
               sa_idx_override=None, out_pad: int = 64) -> Batch:
    """Synthesise one batch of n packets.

    layout="slots": slot stride 2048, headroom 128 -> in_off = 2048 i + 142
    (≡ 14 mod 16, deliberately unaligned), same formula for out_off in a
    separate pool.  layout="packed": datagrams back to back (for host I/O),
    output slots of D + out_pad bytes (out_pad >= 53, the largest ESP overhead).
    locality=k: SA chosen per run of k consecutive packets (flow locality)."""
    r = rng_for(cfg_id, rank, batch)
    L = frame_sizes(n, size, r)
    D = (L.astype(np.int64) - ETH)
    if in_len_override is not None:
        D = np.asarray(in_len_override, np.int64)
        assert D.shape == (n,)
    Dc = np.clip(D, 0, SLOT - HEADROOM - ETH)
    runs = (n + locality - 1) // max(locality, 1)
    sa = np.repeat(r.integers(0, max(n_sa, 1), runs, dtype=np.int64), locality)[:n]
    if sa_idx_override is not None:
        sa = np.asarray(sa_idx_override, np.int64)
    if layout == "slots":
        in_off = (SLOT * np.arange(n, dtype=np.int64) + HEADROOM + ETH)
        out_off = in_off.copy()
        pool = SLOT * max(n, 1)
        out_pool = pool
    elif layout == "packed":
        in_off = np.concatenate([[0], np.cumsum(Dc)[:-1]]) if n else np.zeros(0, np.int64)
        pool = int(Dc.sum()) + 16
        cap = Dc + out_pad
        out_off = np.concatenate([[0], np.cumsum(cap)[:-1]]) if n else np.zeros(0, np.int64)
        out_pool = int(cap.sum()) + 16
    else:
        raise ValueError(layout)

    buf = np.zeros(pool, np.uint8)
    if n:
        maxD = int(Dc.max())
        # random datagram bytes, then overwrite the IPv4/UDP headers
        pk = r.integers(0, 256, (n, max(maxD, 28)), dtype=np.uint8)
        hdr = np.zeros((n, 28), np.uint8)
        hdr[:, 0] = 0x45
        hdr[:, 1] = 0                                    # TOS 0
        hdr[:, 2] = (Dc >> 8) & 0xFF
        hdr[:, 3] = Dc & 0xFF
        hdr[:, 4:6] = r.integers(0, 256, (n, 2), dtype=np.uint8)   # ID
        hdr[:, 6] = 0x40                                 # DF
        hdr[:, 8] = 64                                   # TTL
        hdr[:, 9] = 17                                   # UDP
        hdr[:, 12] = 10
        hdr[:, 13:16] = r.integers(0, 256, (n, 3), dtype=np.uint8)
        hdr[:, 16] = 10
        hdr[:, 17:20] = r.integers(0, 256, (n, 3), dtype=np.uint8)
        words = (hdr[:, 0:20:2].astype(np.uint32) << 8) | hdr[:, 1:20:2]
        cs = _csum16(words)
        hdr[:, 10] = cs >> 8
        hdr[:, 11] = cs & 0xFF
        ports = r.integers(1024, 65536, (n, 2), dtype=np.int64)
        hdr[:, 20] = ports[:, 0] >> 8
        hdr[:, 21] = ports[:, 0] & 0xFF
        hdr[:, 22] = ports[:, 1] >> 8
        hdr[:, 23] = ports[:, 1] & 0xFF
        ulen = np.clip(Dc - 20, 0, 65535)
        hdr[:, 24] = (ulen >> 8) & 0xFF
        hdr[:, 25] = ulen & 0xFF
        pk[:, :28] = hdr
        W = pk.shape[1]
        mask = np.arange(W)[None, :] < Dc[:, None]
        if layout == "slots":
            pool2d = buf.reshape(n, SLOT)
            view = pool2d[:, HEADROOM + ETH:HEADROOM + ETH + W]
            view[mask[:, :view.shape[1]]] = pk[:, :view.shape[1]][mask[:, :view.shape[1]]]
            # Ethernet header in front of the datagram (random MACs, type 0x0800)
            eth = r.integers(0, 256, (n, ETH), dtype=np.uint8)
            eth[:, 12] = 0x08
            eth[:, 13] = 0x00
            pool2d[:, HEADROOM:HEADROOM + ETH] = eth
        else:
            flat = pk[mask]                                  # row-major = back to back
            buf[:flat.size] = flat
    return Batch(n=n, in_buf=buf, in_off=in_off.astype(np.uint32),
                 in_len=np.asarray(D, np.int64).astype(np.uint16), sa_idx=sa.astype(np.uint32),
                 out_off=out_off.astype(np.uint32), out_pool_bytes=int(out_pool),
                 frame_len=L.astype(np.uint32))


# BASELINE.json configs, in order (configs[0..4]).
CONFIGS = {
    1: dict(name="c1_64x64B_1sa", n=64, size=64, n_sa=1),
    2: dict(name="c2_64B_1024sa", n=65536, size=64, n_sa=1024),
    3: dict(name="c3_1514B_1024sa", n=65536, size=1514, n_sa=1024),
    4: dict(name="c4_imix_1024sa", n=65536, size="imix", n_sa=1024),
}
SWEEP_SIZES = (64, 128, 256, 512, 1024, 1514, "imix")   # configs[4]


# --- inbound (ESP decapsulation) traffic -------------------
# An inbound batch is a sequence of ESP tunnel packets.  They are produced by an
# OUTBOUND run (the oracle's in tests, the library's own in bench.py); this
# module only rearranges those bytes -- arrival order, replays, corruption --
# and holds no ESP arithmetic.

def arrival_order(n_src: int, n: int, r: np.random.Generator, reorder: int = 0,
                  dup: float = 0.0, old: float = 0.0, old_span: int = 4096) -> np.ndarray:
    """Indices into the source packets for n arrivals: the source order, with
    local reordering inside windows of `reorder` packets, a fraction `dup`
    replaced by a recent earlier arrival (replayed duplicates) and a fraction
    `old` by one from up to `old_span` arrivals back (stale replays)."""
    idx = np.arange(n, dtype=np.int64) % max(n_src, 1)
    if reorder > 1:
        for s in range(0, n, reorder):
            seg = idx[s:s + reorder]
            idx[s:s + reorder] = seg[r.permutation(seg.size)]
    pos = np.arange(n, dtype=np.int64)
    u = r.random(n)
    d = (u < dup) & (pos > 0)
    idx[d] = idx[pos[d] - r.integers(1, 1 + np.minimum(pos[d], 256))]
    o = (u >= dup) & (u < dup + old) & (pos > 0)
    idx[o] = idx[pos[o] - r.integers(1, 1 + np.minimum(pos[o], old_span))]
    return idx


def esp_batch(src_buf: np.ndarray, src_off: np.ndarray, src_len: np.ndarray,
              src_sa: np.ndarray, order: np.ndarray, corrupt: float = 0.0,
              r: np.random.Generator | None = None, layout: str = "slots") -> Batch:
    """Inbound batch whose packet j is source packet order[j] copied verbatim
    (slot layout as make_batch: in_off = 2048 j + 142, same for out_off).  A
    fraction `corrupt` of the packets gets one random byte XOR-ed with a random
    nonzero value.  frame_len = in_len + 14 (Ethernet, reading A2)."""
    order = np.asarray(order, np.int64)
    n = int(order.size)
    L = np.asarray(src_len, np.int64)[order]
    if layout == "slots":
        in_off = SLOT * np.arange(n, dtype=np.int64) + HEADROOM + ETH
        pool = SLOT * max(n, 1)
        out_off, out_pool = in_off.copy(), pool
    elif layout == "packed":
        in_off = np.concatenate([[0], np.cumsum(L)[:-1]]) if n else np.zeros(0, np.int64)
        pool = int(L.sum()) + 16
        out_off, out_pool = in_off.copy(), pool
    else:
        raise ValueError(layout)
    buf = np.zeros(pool, np.uint8)
    so = np.asarray(src_off, np.int64)[order]
    for j in range(n):
        buf[in_off[j]:in_off[j] + L[j]] = src_buf[so[j]:so[j] + L[j]]
    if corrupt > 0 and n:
        r = r if r is not None else rng_for(0, salt=7)
        hit = np.nonzero(r.random(n) < corrupt)[0]
        for j in hit:
            if L[j] > 0:
                buf[in_off[j] + int(r.integers(0, L[j]))] ^= np.uint8(r.integers(1, 256))
    return Batch(n=n, in_buf=buf, in_off=in_off.astype(np.uint32), in_len=L.astype(np.uint16),
                 sa_idx=np.asarray(src_sa, np.int64)[order].astype(np.uint32),
                 out_off=out_off.astype(np.uint32), out_pool_bytes=int(out_pool),
                 frame_len=(L + ETH).astype(np.uint32))


# --- flows (flow -> SA lookup) -------------------------------

@dataclasses.dataclass
class Flows:
    """Exact-match 5-tuple -> SA table (host order; ports 0 for portless protocols)."""
    src: np.ndarray     # u32[n]
    dst: np.ndarray     # u32[n]
    sport: np.ndarray   # u16[n]
    dport: np.ndarray   # u16[n]
    proto: np.ndarray   # u8[n]
    sa: np.ndarray      # u32[n]


def make_flows(n_flows: int, n_sa: int, cfg_id: int = 0, rank: int = 0) -> Flows:
    """n_flows distinct UDP/TCP flows in 10.0.0.0/8, each bound to a random SA
    (per-flow contexts initialised at startup)."""
    r = rng_for(cfg_id, rank, 0, salt=21)
    seen, rows = set(), []
    while len(rows) < n_flows:
        k = int(n_flows - len(rows))
        src = (10 << 24) | r.integers(0, 1 << 24, k)
        dst = (10 << 24) | r.integers(0, 1 << 24, k)
        sp = r.integers(1024, 65536, k)
        dp = r.integers(1, 65536, k)
        pr = np.where(r.random(k) < 0.8, 17, 6)
        for t in zip(src.tolist(), dst.tolist(), sp.tolist(), dp.tolist(), pr.tolist()):
            if t not in seen:
                seen.add(t)
                rows.append(t)
    a = np.array(rows[:n_flows], dtype=np.int64).reshape(-1, 5)
    return Flows(src=a[:, 0].astype(np.uint32), dst=a[:, 1].astype(np.uint32),
                 sport=a[:, 2].astype(np.uint16), dport=a[:, 3].astype(np.uint16),
                 proto=a[:, 4].astype(np.uint8),
                 sa=r.integers(0, max(n_sa, 1), n_flows).astype(np.uint32))


def apply_flows(b: Batch, flows: Flows, cfg_id: int = 0, batch: int = 0, miss: float = 0.0) -> np.ndarray:
    """Rewrite the inner IPv4 / TCP-UDP headers of every packet of ``b`` (slot
    layout) to a random flow of ``flows``; a fraction ``miss`` gets an unknown
    source address.  Keeps the IPv4 checksum valid.  Returns the flow index per
    packet (-1 for a miss).  Input synthesis only: no lookup logic."""
    r = rng_for(cfg_id, 0, batch, salt=22)
    n = int(b.n)
    fi = r.integers(0, len(flows.sa), n)
    is_miss = r.random(n) < miss
    for i in range(n):
        D = int(b.in_len[i])
        if D < 24:
            continue
        o = int(b.in_off[i])
        k = int(fi[i])
        P = b.in_buf[o:o + D]
        src = int(flows.src[k]) if not is_miss[i] else (11 << 24) | int(r.integers(0, 1 << 24))
        P[12:16] = np.frombuffer(src.to_bytes(4, "big"), np.uint8)
        P[16:20] = np.frombuffer(int(flows.dst[k]).to_bytes(4, "big"), np.uint8)
        P[9] = int(flows.proto[k])
        P[20:22] = np.frombuffer(int(flows.sport[k]).to_bytes(2, "big"), np.uint8)
        P[22:24] = np.frombuffer(int(flows.dport[k]).to_bytes(2, "big"), np.uint8)
        P[10:12] = 0
        words = (P[0:20:2].astype(np.uint32) << 8) | P[1:20:2]
        cs = int(_csum16(words[None, :])[0])
        P[10], P[11] = cs >> 8, cs & 0xFF
    return np.where(is_miss, -1, fi)
