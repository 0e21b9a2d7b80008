"""Thin ctypes binding of libnba_ipsec.so (include/nba_ipsec.h).

Argument marshalling only: every step of the ESP path runs in the library's
CUDA kernels.  PyTorch supplies device memory (tensors' data_ptr) and streams.
There is no CPU fallback: if the library is missing, importing this module
raises.  Names follow the C ABI (nba_ipsec_create_sa_table /
nba_ipsec_process_batch / nba_ipsec_destroy ...).
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# NBA_IPSEC_LIB: an A/B build variant of the same library (tools/ring_ab.py)
LIB_PATH = os.environ.get("NBA_IPSEC_LIB") or os.path.join(_HERE, "libnba_ipsec.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "nba_ipsec.h")

OK, EINVAL, ENOMEM, ENODEV, ECUDA = 0, -22, -12, -19, -1000
PIPE_FUSED, PIPE_UNFUSED = 0, 1
MIN_DATAGRAM, MAX_DATAGRAM, MAX_OVERHEAD = 20, 1500, 53
IN_OK, IN_DROP_SA, IN_DROP_FORMAT, IN_DROP_REPLAY, IN_DROP_AUTH, IN_DROP_TRAILER = range(6)
REPLAY_WINDOW = 64


class NbaIpsecError(RuntimeError):
    def __init__(self, code, what):
        super().__init__(f"{what}: {strerror(code)} ({code})")
        self.code = code


class SaParams(ctypes.Structure):
    _fields_ = [("spi", ctypes.c_uint32), ("tunnel_src", ctypes.c_uint32),
                ("tunnel_dst", ctypes.c_uint32), ("aes_key", ctypes.c_uint8 * 16),
                ("ctr_nonce", ctypes.c_uint8 * 4), ("hmac_key", ctypes.c_uint8 * 20),
                ("seq", ctypes.c_uint32)]


class Batch(ctypes.Structure):
    _fields_ = [("in_buf", ctypes.c_void_p), ("in_off", ctypes.c_void_p),
                ("in_len", ctypes.c_void_p), ("sa_idx", ctypes.c_void_p),
                ("out_buf", ctypes.c_void_p), ("out_off", ctypes.c_void_p),
                ("out_len", ctypes.c_void_p), ("n_pkts", ctypes.c_uint32)]


class Counters(ctypes.Structure):
    _fields_ = [("pkts_ok", ctypes.c_uint64), ("pkts_dropped", ctypes.c_uint64),
                ("bytes_in", ctypes.c_uint64), ("bytes_out", ctypes.c_uint64),
                ("batches", ctypes.c_uint64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


NO_SA = 0xFFFFFFFF


class Flow(ctypes.Structure):
    _fields_ = [("src", ctypes.c_uint32), ("dst", ctypes.c_uint32), ("sport", ctypes.c_uint16),
                ("dport", ctypes.c_uint16), ("proto", ctypes.c_uint8), ("pad_", ctypes.c_uint8 * 3),
                ("sa", ctypes.c_uint32)]


class AlbParams(ctypes.Structure):
    _fields_ = [("steps", ctypes.c_uint32), ("init_step", ctypes.c_uint32),
                ("history", ctypes.c_uint32), ("update_ns", ctypes.c_uint64),
                ("wait_min", ctypes.c_uint32), ("wait_max", ctypes.c_uint32)]


ALB_MAX_DEV, ALB_TREE_NODES = 8, 15


class InBatch(ctypes.Structure):
    _fields_ = [("in_buf", ctypes.c_void_p), ("in_off", ctypes.c_void_p),
                ("in_len", ctypes.c_void_p), ("sa_idx", ctypes.c_void_p),
                ("out_buf", ctypes.c_void_p), ("out_off", ctypes.c_void_p),
                ("out_len", ctypes.c_void_p), ("status", ctypes.c_void_p),
                ("n_pkts", ctypes.c_uint32)]


class InCounters(ctypes.Structure):
    _fields_ = [("pkts_ok", ctypes.c_uint64), ("drop_sa", ctypes.c_uint64),
                ("drop_format", ctypes.c_uint64), ("drop_replay", ctypes.c_uint64),
                ("drop_auth", ctypes.c_uint64), ("drop_trailer", ctypes.c_uint64),
                ("bytes_in", ctypes.c_uint64), ("bytes_out", ctypes.c_uint64),
                ("batches", ctypes.c_uint64)]

    def as_dict(self):
        return {k: int(getattr(self, k)) for k, _ in self._fields_}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -m "
                          "paper_conf_eurosys_kimjlmsm15_b200.build` (no CPU fallback exists)")
    L = ctypes.CDLL(LIB_PATH)
    P = ctypes.POINTER
    vp, i32, u32, u64 = ctypes.c_void_p, ctypes.c_int, ctypes.c_uint32, ctypes.c_uint64
    sig = {
        "nba_ipsec_create_sa_table": (i32, [P(SaParams), u32, i32, u32, P(vp)]),
        "nba_ipsec_process_batch": (i32, [vp, P(Batch), vp]),
        "nba_ipsec_process_batch_host": (i32, [vp, P(Batch), u64, u64, vp]),
        "nba_ipsec_reserve_host_io": (i32, [vp, u64, u64]),
        "nba_ipsec_host_wait": (i32, [vp, vp]),
        "nba_ipsec_destroy": (i32, [vp]),
        "nba_ipsec_read_counters": (i32, [vp, P(Counters), vp]),
        "nba_ipsec_read_sa_seq": (i32, [vp, P(u32), vp]),
        "nba_ipsec_strerror": (ctypes.c_char_p, [i32]),
        "nba_ipsec_set_pipeline": (i32, [vp, i32]),
        "nba_ipsec_launches_per_batch": (i32, [vp]),
        "nba_ipsec_inbound_launches_per_batch": (i32, [vp]),
        "nba_ipsec_profile_enable": (i32, [vp, i32]),
        "nba_ipsec_profile_read": (i32, [vp, P(ctypes.c_double), P(ctypes.c_char_p), i32,
                                         P(i32), P(u32)]),
        "nba_ipsec_debug_trace": (i32, [vp, P(u64), u32]),
        "nba_ipsec_enable_inbound": (i32, [vp]),
        "nba_ipsec_set_flow_table": (i32, [vp, P(Flow), u32]),
        "nba_ipsec_route_workspace_bytes": (i32, [u32, u32, P(u64)]),
        "nba_ipsec_route_pack": (i32, [vp, vp, vp, vp, u32, u32, u32, vp, vp, vp, vp, vp, vp, vp]),
        "nba_ipsec_route_pack_map": (i32, [vp, vp, vp, vp, u32, u32, vp, u32, vp, vp, vp, vp, vp, vp,
                                           vp]),
        "nba_ipsec_write_sa_seq": (i32, [vp, P(u32), vp]),
        "nba_ipsec_route_dispatch": (i32, [vp, vp, vp, vp, u32, u32, vp, u32, vp, vp, u64, u64, vp,
                                           vp, vp]),
        "nba_ipsec_ring_create": (i32, [vp, P(Batch), u32, P(vp)]),
        "nba_ipsec_ring_run": (i32, [vp, u32, vp]),
        "nba_ipsec_ring_run_batches": (i32, [vp, u32, vp]),
        "nba_ipsec_ring_cursor": (i32, [vp]),
        "nba_ipsec_ring_set_timestamps": (i32, [vp, vp, u32]),
        "nba_ipsec_ring_form": (i32, [vp]),
        "nba_ipsec_ring_set_form": (i32, [vp, i32]),
        "nba_ipsec_ring_create_inbound": (i32, [vp, P(InBatch), u32, P(vp)]),
        "nba_ipsec_ring_destroy": (i32, [vp]),
        "nba_ipsec_alb_default_params": (None, [P(AlbParams)]),
        "nba_ipsec_alb_create": (i32, [P(AlbParams), P(vp)]),
        "nba_ipsec_alb_observe": (i32, [vp, u64, u64, u64, P(u32)]),
        "nba_ipsec_alb_state": (i32, [vp, P(u32), P(i32), P(u64)]),
        "nba_ipsec_alb_destroy": (i32, [vp]),
        "nba_ipsec_alb_assign": (i32, [u32, u32, P(u32), u32, P(u32), P(u32)]),
        "nba_ipsec_lookup_sa": (i32, [vp, vp, vp, vp, u32, vp, vp]),
        "nba_ipsec_process_inbound": (i32, [vp, P(InBatch), vp]),
        "nba_ipsec_read_in_counters": (i32, [vp, P(InCounters), vp]),
        "nba_ipsec_reset_inbound": (i32, [vp, vp]),
        "nba_ipsec_read_replay_window": (i32, [vp, P(u32), P(u64), vp]),
        "nba_ipsec_profile_read_inbound": (i32, [vp, P(ctypes.c_double), P(ctypes.c_char_p), i32,
                                                 P(i32), P(u32)]),
        "nba_ipsec_host_aes128_key_schedule": (None, [P(ctypes.c_uint8), P(u32)]),
        "nba_ipsec_host_hmac_sha1_midstates": (None, [P(ctypes.c_uint8), P(u32), P(u32)]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    return L


lib = _load()


def header_functions() -> list[str]:
    """Function names declared in include/nba_ipsec.h."""
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"\b(nba_ipsec_[a-z0-9_]+)\s*\(", txt)))


def strerror(code: int) -> str:
    return lib.nba_ipsec_strerror(int(code)).decode()


def _check(rc, what):
    if rc != OK:
        raise NbaIpsecError(rc, what)


def make_params(p) -> "ctypes.Array":
    """gen.SAParams (numpy SoA) -> nba_ipsec_sa_params[n]."""
    n = len(p.spi)
    arr = (SaParams * max(n, 1))()
    for s in range(n):
        e = arr[s]
        e.spi = int(p.spi[s])
        e.tunnel_src = int(p.tunnel_src[s])
        e.tunnel_dst = int(p.tunnel_dst[s])
        ctypes.memmove(e.aes_key, np.ascontiguousarray(p.aes_key[s], np.uint8).ctypes.data, 16)
        ctypes.memmove(e.ctr_nonce, np.ascontiguousarray(p.ctr_nonce[s], np.uint8).ctypes.data, 4)
        ctypes.memmove(e.hmac_key, np.ascontiguousarray(p.hmac_key[s], np.uint8).ctypes.data, 20)
        e.seq = int(p.seq[s])
    return arr


def _stream_handle(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


def _ptr(x):
    if x is None:
        return None
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return int(x)


class SATable:
    """nba_ipsec_sa_table: per-device SA state + workspace."""

    def __init__(self, params, device: int = 0, max_batch: int = 65536):
        arr = params if isinstance(params, ctypes.Array) else make_params(params)
        self.n_sa = len(params.spi) if not isinstance(params, ctypes.Array) else len(arr)
        self.device = device
        self.max_batch = max_batch
        h = ctypes.c_void_p()
        _check(lib.nba_ipsec_create_sa_table(arr, self.n_sa, device, max_batch, ctypes.byref(h)),
               "nba_ipsec_create_sa_table")
        self._h = h

    # -- hot path ------------------------------------------------------------
    def process(self, in_buf, in_off, in_len, sa_idx, out_buf, out_off, out_len, n=None,
                stream=None):
        """nba_ipsec_process_batch on device tensors (uint8 / int32 / int16 views)."""
        n = int(in_len.numel() if n is None else n)
        b = Batch(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_idx), _ptr(out_buf),
                  _ptr(out_off), _ptr(out_len), n)
        _check(lib.nba_ipsec_process_batch(self._h, ctypes.byref(b), _stream_handle(stream)),
               "nba_ipsec_process_batch")

    def reserve_host_io(self, in_bytes: int, out_bytes: int):
        _check(lib.nba_ipsec_reserve_host_io(self._h, in_bytes, out_bytes),
               "nba_ipsec_reserve_host_io")

    def process_host(self, in_buf, in_off, in_len, sa_idx, out_buf, out_off, out_len,
                     in_bytes, out_bytes, n=None, stream=None):
        """nba_ipsec_process_batch_host on host (pinned) buffers."""
        n = int(len(in_len) if n is None else n)
        b = Batch(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_idx), _ptr(out_buf),
                  _ptr(out_off), _ptr(out_len), n)
        _check(lib.nba_ipsec_process_batch_host(self._h, ctypes.byref(b), int(in_bytes),
                                                int(out_bytes), _stream_handle(stream)),
               "nba_ipsec_process_batch_host")

    def host_wait(self, stream=None):
        """nba_ipsec_host_wait: `stream` waits for every host-path batch's outputs."""
        _check(lib.nba_ipsec_host_wait(self._h, _stream_handle(stream)), "nba_ipsec_host_wait")

    # -- auxiliary -------------------------------------------------------------
    def counters(self, stream=None) -> dict:
        c = Counters()
        _check(lib.nba_ipsec_read_counters(self._h, ctypes.byref(c), _stream_handle(stream)),
               "nba_ipsec_read_counters")
        return c.as_dict()

    def sa_seq(self, stream=None) -> np.ndarray:
        out = np.zeros(self.n_sa, np.uint32)
        _check(lib.nba_ipsec_read_sa_seq(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                                         _stream_handle(stream)), "nba_ipsec_read_sa_seq")
        return out

    def write_sa_seq(self, seq, stream=None):
        """nba_ipsec_write_sa_seq: replace every SA's counter (hand-over, L7)."""
        a = np.ascontiguousarray(seq, dtype=np.uint32)
        if a.shape != (self.n_sa,):
            raise ValueError(f"need {self.n_sa} sequence numbers")
        _check(lib.nba_ipsec_write_sa_seq(self._h, a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                                          _stream_handle(stream)), "nba_ipsec_write_sa_seq")

    def ring(self, slots):
        """nba_ipsec_ring_create: `slots` = sequence of (in_buf, in_off, in_len,
        sa_idx, out_buf, out_off, out_len, n) device-tensor tuples."""
        return Ring(self, slots)

    def ring_inbound(self, slots):
        """nba_ipsec_ring_create_inbound: `slots` = sequence of (in_buf, in_off,
        in_len, sa_idx, out_buf, out_off, out_len, status-or-None, n)."""
        return Ring(self, slots, inbound=True)

    def set_pipeline(self, pipeline: int):
        _check(lib.nba_ipsec_set_pipeline(self._h, int(pipeline)), "nba_ipsec_set_pipeline")

    def launches_per_batch(self) -> int:
        return int(lib.nba_ipsec_launches_per_batch(self._h))

    def inbound_launches_per_batch(self) -> int:
        return int(lib.nba_ipsec_inbound_launches_per_batch(self._h))

    def profile_enable(self, on: bool = True):
        _check(lib.nba_ipsec_profile_enable(self._h, 1 if on else 0), "nba_ipsec_profile_enable")

    def profile_read(self) -> tuple[dict, int]:
        ms = (ctypes.c_double * 8)()
        names = (ctypes.c_char_p * 8)()
        nk, nb = ctypes.c_int(0), ctypes.c_uint32(0)
        _check(lib.nba_ipsec_profile_read(self._h, ms, names, 8, ctypes.byref(nk),
                                          ctypes.byref(nb)), "nba_ipsec_profile_read")
        return {names[k].decode(): ms[k] for k in range(nk.value)}, int(nb.value)

    # -- flow -> SA lookup ------------------------------------
    def set_flow_table(self, flows):
        """nba_ipsec_set_flow_table from a gen.Flows (numpy SoA)."""
        n = len(flows.sa)
        arr = (Flow * max(n, 1))()
        for k in range(n):
            f = arr[k]
            f.src, f.dst = int(flows.src[k]), int(flows.dst[k])
            f.sport, f.dport, f.proto = int(flows.sport[k]), int(flows.dport[k]), int(flows.proto[k])
            f.sa = int(flows.sa[k])
        _check(lib.nba_ipsec_set_flow_table(self._h, arr, n), "nba_ipsec_set_flow_table")

    def lookup_sa(self, in_buf, in_off, in_len, sa_idx, n=None, stream=None):
        n = int(in_len.numel() if n is None else n)
        _check(lib.nba_ipsec_lookup_sa(self._h, _ptr(in_buf), _ptr(in_off), _ptr(in_len), n,
                                       _ptr(sa_idx), _stream_handle(stream)), "nba_ipsec_lookup_sa")

    # -- ESP inbound ------------------------------------------
    def enable_inbound(self):
        _check(lib.nba_ipsec_enable_inbound(self._h), "nba_ipsec_enable_inbound")

    def process_inbound(self, in_buf, in_off, in_len, sa_idx, out_buf, out_off, out_len,
                        status=None, n=None, stream=None):
        """nba_ipsec_process_inbound on device tensors; status (uint8) optional."""
        n = int(in_len.numel() if n is None else n)
        b = InBatch(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_idx), _ptr(out_buf),
                    _ptr(out_off), _ptr(out_len), _ptr(status), n)
        _check(lib.nba_ipsec_process_inbound(self._h, ctypes.byref(b), _stream_handle(stream)),
               "nba_ipsec_process_inbound")

    def reset_inbound(self, stream=None):
        _check(lib.nba_ipsec_reset_inbound(self._h, _stream_handle(stream)),
               "nba_ipsec_reset_inbound")

    def in_counters(self, stream=None) -> dict:
        c = InCounters()
        _check(lib.nba_ipsec_read_in_counters(self._h, ctypes.byref(c), _stream_handle(stream)),
               "nba_ipsec_read_in_counters")
        return c.as_dict()

    def replay_window(self, stream=None):
        top = np.zeros(self.n_sa, np.uint32)
        bmp = np.zeros(self.n_sa, np.uint64)
        _check(lib.nba_ipsec_read_replay_window(
            self._h, top.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
            bmp.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), _stream_handle(stream)),
            "nba_ipsec_read_replay_window")
        return top, bmp

    def profile_read_inbound(self) -> tuple[dict, int]:
        ms = (ctypes.c_double * 3)()
        names = (ctypes.c_char_p * 3)()
        nk, nb = ctypes.c_int(0), ctypes.c_uint32(0)
        _check(lib.nba_ipsec_profile_read_inbound(self._h, ms, names, 3, ctypes.byref(nk),
                                                  ctypes.byref(nb)),
               "nba_ipsec_profile_read_inbound")
        return {names[k].decode(): ms[k] for k in range(nk.value)}, int(nb.value)

    def debug_trace(self, n_cta: int = 148) -> np.ndarray:
        """(n_cta + 1, 8) timestamps; the last row is the prologue's."""
        out = np.zeros(n_cta * 8 + 8, np.uint64)
        _check(lib.nba_ipsec_debug_trace(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)),
                                         out.size), "nba_ipsec_debug_trace")
        return out.reshape(n_cta + 1, 8)

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            _check(lib.nba_ipsec_destroy(self._h), "nba_ipsec_destroy")
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


# -- host-only setup helpers (tests of the library's own a0 arithmetic) ---------
def host_aes128_key_schedule(key: bytes) -> np.ndarray:
    k = np.frombuffer(bytes(key), np.uint8).copy()
    w = np.zeros(44, np.uint32)
    lib.nba_ipsec_host_aes128_key_schedule(k.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
                                           w.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    return w


def host_hmac_sha1_midstates(key: bytes):
    k = np.frombuffer(bytes(key), np.uint8).copy()
    hin, hout = np.zeros(5, np.uint32), np.zeros(5, np.uint32)
    u32p = ctypes.POINTER(ctypes.c_uint32)
    lib.nba_ipsec_host_hmac_sha1_midstates(k.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)),
                                           hin.ctypes.data_as(u32p), hout.ctypes.data_as(u32p))
    return hin, hout


# -- single-ingress redistribution ----------------------------
def route_workspace_bytes(max_pkts: int, world: int) -> int:
    b = ctypes.c_uint64(0)
    _check(lib.nba_ipsec_route_workspace_bytes(max_pkts, world, ctypes.byref(b)),
           "nba_ipsec_route_workspace_bytes")
    return int(b.value)


def route_pack(in_buf, in_off, in_len, sa_global, n, n_sa_total, world, workspace, send_buf,
               send_len, send_sa, dest_counts, dest_bytes, stream=None):
    """nba_ipsec_route_pack on device tensors (see include/nba_ipsec.h)."""
    _check(lib.nba_ipsec_route_pack(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_global), int(n),
                                    int(n_sa_total), int(world), _ptr(workspace), _ptr(send_buf),
                                    _ptr(send_len), _ptr(send_sa), _ptr(dest_counts),
                                    _ptr(dest_bytes), _stream_handle(stream)),
           "nba_ipsec_route_pack")


def route_pack_map(in_buf, in_off, in_len, sa_global, n, n_sa_total, sa_map, world, workspace,
                   send_buf, send_len, send_sa, dest_counts, dest_bytes, stream=None):
    """nba_ipsec_route_pack_map: routing by an explicit owner map (f4)."""
    _check(lib.nba_ipsec_route_pack_map(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_global),
                                        int(n), int(n_sa_total), _ptr(sa_map), int(world),
                                        _ptr(workspace), _ptr(send_buf), _ptr(send_len),
                                        _ptr(send_sa), _ptr(dest_counts), _ptr(dest_bytes),
                                        _stream_handle(stream)),
           "nba_ipsec_route_pack_map")


class Ring:
    """A fixed set of batch slots recorded as one CUDA graph (nba_ipsec_ring_*)."""

    def __init__(self, table, slots, inbound=False):
        kind = InBatch if inbound else Batch
        arr = (kind * len(slots))()
        self._keep = list(slots)            # the tensors must outlive the ring
        for i, sl in enumerate(slots):
            *bufs, n = sl
            arr[i] = kind(*(_ptr(x) for x in bufs), int(n))
        self.table = table
        self.n_slots = len(slots)
        self._h = ctypes.c_void_p()
        create = lib.nba_ipsec_ring_create_inbound if inbound else lib.nba_ipsec_ring_create
        _check(create(table._h, arr, len(slots), ctypes.byref(self._h)), "nba_ipsec_ring_create")

    def run(self, n_rounds: int = 1, stream=None):
        _check(lib.nba_ipsec_ring_run(self._h, int(n_rounds), _stream_handle(stream)),
               "nba_ipsec_ring_run")

    def run_batches(self, n_batches: int, stream=None):
        """nba_ipsec_ring_run_batches: exactly n_batches batches from the cursor."""
        _check(lib.nba_ipsec_ring_run_batches(self._h, int(n_batches), _stream_handle(stream)),
               "nba_ipsec_ring_run_batches")

    @property
    def cursor(self) -> int:
        return int(lib.nba_ipsec_ring_cursor(self._h))

    def set_timestamps(self, ts):
        """nba_ipsec_ring_set_timestamps: ts = int64 CUDA tensor (cap entries) or None."""
        self._ts = ts
        _check(lib.nba_ipsec_ring_set_timestamps(self._h, _ptr(ts) if ts is not None else None,
                                                 int(ts.numel()) if ts is not None else 0),
               "nba_ipsec_ring_set_timestamps")

    GRAPH, PERSISTENT, PIPELINED, FREE, ROLES = 0, 1, 2, 3, 4

    @property
    def form(self) -> int:
        return int(lib.nba_ipsec_ring_form(self._h))

    def set_form(self, form: int):
        _check(lib.nba_ipsec_ring_set_form(self._h, int(form)), "nba_ipsec_ring_set_form")

    def close(self):
        if self._h:
            lib.nba_ipsec_ring_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def route_dispatch(in_buf, in_off, in_len, sa_global, n, n_sa_total, sa_map, world, workspace,
                   rx_table, cap_pkts, cap_bytes, dest_counts, dest_bytes, stream=None):
    """nba_ipsec_route_dispatch: route + write straight into the owners' receive
    buffers (rx_table: device array of nba_ipsec_peer_rx descriptors)."""
    _check(lib.nba_ipsec_route_dispatch(_ptr(in_buf), _ptr(in_off), _ptr(in_len), _ptr(sa_global),
                                        int(n), int(n_sa_total), _ptr(sa_map), int(world),
                                        _ptr(workspace), _ptr(rx_table), int(cap_pkts),
                                        int(cap_bytes), _ptr(dest_counts), _ptr(dest_bytes),
                                        _stream_handle(stream)),
           "nba_ipsec_route_dispatch")


# -- adaptive split of the SAs across devices -----------------
def alb_default_params() -> AlbParams:
    p = AlbParams()
    lib.nba_ipsec_alb_default_params(ctypes.byref(p))
    return p


class Alb:
    """nba_ipsec_alb_* controller (host code in the library)."""

    def __init__(self, steps=None, init_step=None, history=None, update_ns=None, wait_min=None,
                 wait_max=None):
        p = alb_default_params()
        for k, v in (("steps", steps), ("init_step", init_step), ("history", history),
                     ("update_ns", update_ns), ("wait_min", wait_min), ("wait_max", wait_max)):
            if v is not None:
                setattr(p, k, int(v))
        self.params = p
        self._h = ctypes.c_void_p()
        _check(lib.nba_ipsec_alb_create(ctypes.byref(p), ctypes.byref(self._h)), "nba_ipsec_alb_create")

    def observe(self, t_ns: int, dt_ns: int, pkts: int) -> int:
        k = ctypes.c_uint32(0)
        _check(lib.nba_ipsec_alb_observe(self._h, int(t_ns), int(dt_ns), int(pkts), ctypes.byref(k)),
               "nba_ipsec_alb_observe")
        return int(k.value)

    def state(self):
        k, d, u = ctypes.c_uint32(0), ctypes.c_int(0), ctypes.c_uint64(0)
        _check(lib.nba_ipsec_alb_state(self._h, ctypes.byref(k), ctypes.byref(d), ctypes.byref(u)),
               "nba_ipsec_alb_state")
        return int(k.value), int(d.value), int(u.value)

    def close(self):
        if self._h:
            lib.nba_ipsec_alb_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def alb_assign(n_sa: int, n_dev: int, node_step, steps: int):
    """nba_ipsec_alb_assign -> (owner[n_sa], sa_map[n_sa]) as uint32 arrays."""
    u32p = ctypes.POINTER(ctypes.c_uint32)
    ns = np.zeros(ALB_TREE_NODES, np.uint32)
    ns[:len(node_step)] = node_step
    owner = np.zeros(max(n_sa, 1), np.uint32)
    sa_map = np.zeros(max(n_sa, 1), np.uint32)
    _check(lib.nba_ipsec_alb_assign(int(n_sa), int(n_dev), ns.ctypes.data_as(u32p), int(steps),
                                    owner.ctypes.data_as(u32p), sa_map.ctypes.data_as(u32p)),
           "nba_ipsec_alb_assign")
    return owner[:n_sa], sa_map[:n_sa]
