"""CPU oracle for the NBA IPsec ESP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product package
(``paper_conf_eurosys_kimjlmsm15_b200``) never imports it, and the two share no
code: this is a ctypes wrapper around ``oracle.c`` (plain C99, see its header
for the standards it follows, PAPER.md:389 and PAPER.md:395 for the method).

Parity status: every function here is pinned by tests/test_oracle_*.py
(standard vectors, an independent OpenSSL/pyca composition, round trips and
invariants).  The ESP wire format itself is a reading of the RFCs because the
paper is silent on it; against NBA's real wire format the
result is "parity unpinned" (no implementation of NBA exists to compare with).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

MIN_DATAGRAM = 20
MAX_DATAGRAM = 1500


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc -O2, no crypto intrinsics)."""
    src = os.path.join(_HERE, "oracle.c")
    hdr = os.path.join(_HERE, "oracle.h")
    if (not force and os.path.exists(_SO)
            and os.path.getmtime(_SO) >= max(os.path.getmtime(src), os.path.getmtime(hdr))):
        return _SO
    tmp = _SO + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-std=c99", "-O2", "-fPIC", "-shared", "-pthread",
                           "-Wall", "-Wextra", "-o", tmp, src])
    os.replace(tmp, _SO)
    return _SO


class SA(ctypes.Structure):
    _fields_ = [("spi", ctypes.c_uint32), ("tunnel_src", ctypes.c_uint32),
                ("tunnel_dst", ctypes.c_uint32), ("aes_key", ctypes.c_uint8 * 16),
                ("ctr_nonce", ctypes.c_uint8 * 4), ("hmac_key", ctypes.c_uint8 * 20),
                ("seq", ctypes.c_uint32)]


class Counters(ctypes.Structure):
    _fields_ = [("pkts_ok", ctypes.c_uint64), ("pkts_dropped", ctypes.c_uint64),
                ("bytes_in", ctypes.c_uint64), ("bytes_out", ctypes.c_uint64),
                ("batches", ctypes.c_uint64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


IN_OK, IN_DROP_SA, IN_DROP_FORMAT, IN_DROP_REPLAY, IN_DROP_AUTH, IN_DROP_TRAILER = range(6)
REPLAY_WINDOW = 64


class Replay(ctypes.Structure):
    _fields_ = [("top", ctypes.c_uint32), ("pad_", ctypes.c_uint32), ("bitmap", ctypes.c_uint64)]


class InCounters(ctypes.Structure):
    _fields_ = [("pkts_ok", ctypes.c_uint64), ("drop_sa", ctypes.c_uint64),
                ("drop_format", ctypes.c_uint64), ("drop_replay", ctypes.c_uint64),
                ("drop_auth", ctypes.c_uint64), ("drop_trailer", ctypes.c_uint64),
                ("bytes_in", ctypes.c_uint64), ("bytes_out", ctypes.c_uint64),
                ("batches", ctypes.c_uint64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


NO_SA = 0xFFFFFFFF


class Flow(ctypes.Structure):
    _fields_ = [("src", ctypes.c_uint32), ("dst", ctypes.c_uint32), ("sport", ctypes.c_uint16),
                ("dport", ctypes.c_uint16), ("proto", ctypes.c_uint8), ("pad_", ctypes.c_uint8 * 3),
                ("sa", ctypes.c_uint32)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_SO)
            P = ctypes.POINTER
            u8p, u16p, u32p = P(ctypes.c_uint8), P(ctypes.c_uint16), P(ctypes.c_uint32)
            L.oracle_sbox.restype = ctypes.c_uint8
            L.oracle_sbox.argtypes = [ctypes.c_uint8]
            L.oracle_aes128_expand_key.argtypes = [u8p, u8p]
            L.oracle_aes128_encrypt.argtypes = [u8p, u8p, u8p]
            L.oracle_ctr_xcrypt.argtypes = [u8p, u8p, u8p, ctypes.c_size_t, u8p]
            L.oracle_sha1.argtypes = [u8p, ctypes.c_size_t, u8p]
            L.oracle_hmac_sha1.argtypes = [u8p, ctypes.c_size_t, u8p, ctypes.c_size_t, u8p]
            L.oracle_ipv4_checksum.restype = ctypes.c_uint16
            L.oracle_ipv4_checksum.argtypes = [u8p, ctypes.c_size_t]
            L.oracle_esp_encap.restype = ctypes.c_uint32
            L.oracle_esp_encap.argtypes = [P(SA), ctypes.c_uint32, u8p, ctypes.c_uint32, u8p]
            batch_args = [P(SA), ctypes.c_uint32, u8p, u32p, u16p, u32p, u8p, u32p, u16p,
                          ctypes.c_uint32, P(Counters)]
            L.oracle_process_batch.restype = None
            L.oracle_process_batch.argtypes = batch_args
            L.oracle_process_batch_mt.restype = ctypes.c_int
            L.oracle_process_batch_mt.argtypes = batch_args + [ctypes.c_int]
            L.oracle_decap.restype = ctypes.c_int
            L.oracle_decap.argtypes = [P(SA), u8p, ctypes.c_uint32, u8p, u32p, u32p]
            L.oracle_replay_init.restype = None
            L.oracle_replay_init.argtypes = [P(SA), P(Replay)]
            L.oracle_process_inbound.restype = None
            L.oracle_process_inbound.argtypes = [P(SA), P(Replay), ctypes.c_uint32, u8p, u32p, u16p,
                                                 u32p, u8p, u32p, u16p, u8p, ctypes.c_uint32,
                                                 P(InCounters)]
            L.oracle_flow_table_prepare.restype = ctypes.c_int
            L.oracle_flow_table_prepare.argtypes = [P(Flow), ctypes.c_uint32]
            L.oracle_flow_lookup.restype = None
            L.oracle_flow_lookup.argtypes = [P(Flow), ctypes.c_uint32, u8p, u32p, u16p,
                                             ctypes.c_uint32, u32p]
            L.oracle_init()
            _lib = L
    return _lib


def _u8(b):
    a = np.frombuffer(bytes(b), dtype=np.uint8).copy() if not isinstance(b, np.ndarray) else \
        np.ascontiguousarray(b, dtype=np.uint8)
    return a


def _ptr(a, ct=ctypes.c_uint8):
    return a.ctypes.data_as(ctypes.POINTER(ct))


# --- primitives ------------------------------------------------------------

def sbox(x: int) -> int:
    return int(lib().oracle_sbox(x))


def aes128_expand_key(key: bytes) -> bytes:
    k = _u8(key); assert k.size == 16
    w = np.zeros(176, np.uint8)
    lib().oracle_aes128_expand_key(_ptr(k), _ptr(w))
    return w.tobytes()


def aes128_encrypt(key: bytes, block: bytes) -> bytes:
    k, b = _u8(key), _u8(block); assert k.size == 16 and b.size == 16
    o = np.zeros(16, np.uint8)
    lib().oracle_aes128_encrypt(_ptr(k), _ptr(b), _ptr(o))
    return o.tobytes()


def ctr_xcrypt(key: bytes, icb: bytes, data: bytes) -> bytes:
    k, c, d = _u8(key), _u8(icb), _u8(data)
    o = np.zeros(max(d.size, 1), np.uint8)
    lib().oracle_ctr_xcrypt(_ptr(k), _ptr(c), _ptr(d if d.size else o), d.size, _ptr(o))
    return o[:d.size].tobytes()


def sha1(msg: bytes) -> bytes:
    m = _u8(msg)
    o = np.zeros(20, np.uint8)
    lib().oracle_sha1(_ptr(m if m.size else o), m.size, _ptr(o))
    return o.tobytes()


def hmac_sha1(key: bytes, msg: bytes) -> bytes:
    k, m = _u8(key), _u8(msg)
    o = np.zeros(20, np.uint8)
    lib().oracle_hmac_sha1(_ptr(k if k.size else o), k.size, _ptr(m if m.size else o), m.size,
                           _ptr(o))
    return o.tobytes()


def ipv4_checksum(hdr: bytes) -> int:
    h = _u8(hdr)
    return int(lib().oracle_ipv4_checksum(_ptr(h), h.size))


# --- SA tables and batches --------------------------------------------------

def make_sas(params) -> "ctypes.Array":
    """Build an oracle SA array from a gen.SAParams (numpy SoA)."""
    n = len(params.spi)
    arr = (SA * max(n, 1))()
    for s in range(n):
        e = arr[s]
        e.spi = int(params.spi[s])
        e.tunnel_src = int(params.tunnel_src[s])
        e.tunnel_dst = int(params.tunnel_dst[s])
        e.aes_key[:] = [int(x) for x in params.aes_key[s]]
        e.ctr_nonce[:] = [int(x) for x in params.ctr_nonce[s]]
        e.hmac_key[:] = [int(x) for x in params.hmac_key[s]]
        e.seq = int(params.seq[s])
    return arr


def sa_seq(sas, n_sa: int) -> np.ndarray:
    return np.array([sas[s].seq for s in range(n_sa)], dtype=np.uint32)


def esp_encap(sas, s: int, q: int, inner: bytes) -> bytes:
    P = _u8(inner)
    out = np.zeros(P.size + 64, np.uint8)
    L = lib().oracle_esp_encap(ctypes.byref(sas[s]), q, _ptr(P), P.size, _ptr(out))
    return out[:L].tobytes()


def process_batch(sas, n_sa: int, batch, out_pool_bytes: int | None = None,
                  n_threads: int = 1, out_buf: np.ndarray | None = None,
                  counters: Counters | None = None):
    """Run the sequential (n_threads=1) or SA-partitioned threaded oracle.

    ``batch`` is a gen.Batch (numpy arrays).  ``sas`` is updated in place
    (sequence numbers advance).  Returns (out_buf, out_len, counters)."""
    n = int(batch.n)
    in_buf = np.ascontiguousarray(batch.in_buf, np.uint8)
    in_off = np.ascontiguousarray(batch.in_off, np.uint32)
    in_len = np.ascontiguousarray(batch.in_len, np.uint16)
    sa_idx = np.ascontiguousarray(batch.sa_idx, np.uint32)
    out_off = np.ascontiguousarray(batch.out_off, np.uint32)
    if out_buf is None:
        size = out_pool_bytes if out_pool_bytes is not None else batch.out_pool_bytes
        out_buf = np.zeros(max(size, 1), np.uint8)
    out_len = np.zeros(max(n, 1), np.uint16)
    ctr = counters if counters is not None else Counters()
    args = (sas, n_sa, _ptr(in_buf), _ptr(in_off, ctypes.c_uint32), _ptr(in_len, ctypes.c_uint16),
            _ptr(sa_idx, ctypes.c_uint32), _ptr(out_buf), _ptr(out_off, ctypes.c_uint32),
            _ptr(out_len, ctypes.c_uint16), n, ctypes.byref(ctr))
    if n_threads <= 1:
        lib().oracle_process_batch(*args)
    else:
        rc = lib().oracle_process_batch_mt(*args, int(n_threads))
        if rc != 0:
            raise MemoryError("oracle_process_batch_mt failed")
    return out_buf, out_len[:n], ctr


def decap(sas, s: int, pkt: bytes):
    """Inbound check used by tests: returns (rc, inner_bytes, seq)."""
    p = _u8(pkt)
    inner = np.zeros(max(p.size, 1), np.uint8)
    ilen = ctypes.c_uint32(0)
    seq = ctypes.c_uint32(0)
    rc = lib().oracle_decap(ctypes.byref(sas[s]), _ptr(p), p.size, _ptr(inner),
                            ctypes.byref(ilen), ctypes.byref(seq))
    return rc, inner[:ilen.value].tobytes(), seq.value


# --- ESP inbound -------------------------------------------

def make_windows(sas, n_sa: int) -> "ctypes.Array":
    """Per-SA anti-replay windows initialised from the SAs' ``seq`` (reading B6)."""
    arr = (Replay * max(n_sa, 1))()
    for s in range(n_sa):
        lib().oracle_replay_init(ctypes.byref(sas[s]), ctypes.byref(arr[s]))
    return arr


def window_state(win, n_sa: int):
    top = np.array([win[s].top for s in range(n_sa)], dtype=np.uint32)
    bmp = np.array([win[s].bitmap for s in range(n_sa)], dtype=np.uint64)
    return top, bmp


def process_inbound(sas, win, n_sa: int, batch, out_pool_bytes: int | None = None,
                    counters: InCounters | None = None):
    """Sequential ESP inbound over ``batch`` (a gen.Batch whose in_buf holds ESP
    tunnel packets).  ``win`` is updated in place.  Returns
    (out_buf, out_len, status, counters); only out_buf[out_off[i] : +out_len[i]]
    is defined."""
    n = int(batch.n)
    in_buf = np.ascontiguousarray(batch.in_buf, np.uint8)
    in_off = np.ascontiguousarray(batch.in_off, np.uint32)
    in_len = np.ascontiguousarray(batch.in_len, np.uint16)
    sa_idx = np.ascontiguousarray(batch.sa_idx, np.uint32)
    out_off = np.ascontiguousarray(batch.out_off, np.uint32)
    size = out_pool_bytes if out_pool_bytes is not None else batch.out_pool_bytes
    out_buf = np.zeros(max(size, 1), np.uint8)
    out_len = np.zeros(max(n, 1), np.uint16)
    status = np.zeros(max(n, 1), np.uint8)
    ctr = counters if counters is not None else InCounters()
    lib().oracle_process_inbound(sas, win, n_sa, _ptr(in_buf), _ptr(in_off, ctypes.c_uint32),
                                 _ptr(in_len, ctypes.c_uint16), _ptr(sa_idx, ctypes.c_uint32),
                                 _ptr(out_buf), _ptr(out_off, ctypes.c_uint32),
                                 _ptr(out_len, ctypes.c_uint16), _ptr(status), n,
                                 ctypes.byref(ctr))
    return out_buf, out_len[:n], status[:n], ctr


# --- flow -> SA lookup -------------------------------------

def flow_lookup(flows, batch) -> np.ndarray:
    """SA index per packet of ``batch`` from the exact-match 5-tuple table
    ``flows`` (a gen.Flows); NO_SA where there is no key or no match."""
    nf = len(flows.sa)
    arr = (Flow * max(nf, 1))()
    for k in range(nf):
        f = arr[k]
        f.src, f.dst = int(flows.src[k]), int(flows.dst[k])
        f.sport, f.dport, f.proto = int(flows.sport[k]), int(flows.dport[k]), int(flows.proto[k])
        f.sa = int(flows.sa[k])
    if lib().oracle_flow_table_prepare(arr, nf) != 0:
        raise ValueError("duplicate flow keys")
    n = int(batch.n)
    in_buf = np.ascontiguousarray(batch.in_buf, np.uint8)
    in_off = np.ascontiguousarray(batch.in_off, np.uint32)
    in_len = np.ascontiguousarray(batch.in_len, np.uint16)
    out = np.zeros(max(n, 1), np.uint32)
    lib().oracle_flow_lookup(arr, nf, _ptr(in_buf), _ptr(in_off, ctypes.c_uint32),
                             _ptr(in_len, ctypes.c_uint16), n, _ptr(out, ctypes.c_uint32))
    return out[:n]
