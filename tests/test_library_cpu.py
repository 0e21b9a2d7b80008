"""CPU-only checks of the C-ABI library: it loads, exports every symbol the
header declares, validates arguments before touching a device, and its
setup-time (row a0) arithmetic matches FIPS-197 / RFC 2202 (no GPU needed)."""
import ctypes

import numpy as np
import pytest

from golden import load, msg_of
import pysha1

nb = pytest.importorskip("paper_conf_eurosys_kimjlmsm15_b200.nba_ipsec")
AES = load("aes_vectors.txt")
SHA = load("sha1_hmac_vectors.txt")


def test_exports_every_header_symbol():
    names = nb.header_functions()
    assert "nba_ipsec_create_sa_table" in names and "nba_ipsec_process_batch" in names
    assert "nba_ipsec_destroy" in names
    for n in names:
        assert hasattr(nb.lib, n), n


def test_strerror():
    assert nb.strerror(0) == "ok"
    assert "invalid" in nb.strerror(nb.EINVAL)
    assert nb.strerror(12345) == "unknown error"


def test_argument_errors_without_device():
    lib = nb.lib
    h = ctypes.c_void_p()
    arr = (nb.SaParams * 1)()
    assert lib.nba_ipsec_create_sa_table(arr, 1, 0, 64, None) == nb.EINVAL
    assert lib.nba_ipsec_create_sa_table(None, 1, 0, 64, ctypes.byref(h)) == nb.EINVAL
    assert lib.nba_ipsec_create_sa_table(arr, 0, 0, 64, ctypes.byref(h)) == nb.EINVAL
    assert lib.nba_ipsec_create_sa_table(arr, 1, 0, 0, ctypes.byref(h)) == nb.EINVAL
    assert lib.nba_ipsec_create_sa_table(arr, 1 << 17, 0, 64, ctypes.byref(h)) == nb.EINVAL
    assert lib.nba_ipsec_create_sa_table(arr, 1, -1, 64, ctypes.byref(h)) == nb.ENODEV
    assert lib.nba_ipsec_process_batch(None, None, None) == nb.EINVAL
    assert lib.nba_ipsec_destroy(None) == nb.OK
    assert lib.nba_ipsec_read_counters(None, None, None) == nb.EINVAL


def test_host_key_schedule_fips197_a1():
    r = AES["fips197_a1"]
    w = nb.host_aes128_key_schedule(bytes.fromhex(r["key"]))
    assert b"".join(int(x).to_bytes(4, "big") for x in w[4:8]).hex() == r["w4_7"]
    assert b"".join(int(x).to_bytes(4, "big") for x in w[40:44]).hex() == r["w40_43"]


@pytest.mark.parametrize("name", ["rfc2202_1", "rfc2202_3", "rfc2202_5"])
def test_host_hmac_midstates_rfc2202(name):
    """Continuing SHA-1 from the library's ipad/opad midstates reproduces the
    RFC 2202 digests (the 20-byte-key cases the library accepts)."""
    r = SHA[name]
    hin, hout = nb.host_hmac_sha1_midstates(bytes.fromhex(r["key"]))
    inner = pysha1.finish([int(x) for x in hin], msg_of(r), 64)
    outer = pysha1.finish([int(x) for x in hout], inner, 64)
    assert outer.hex() == r["digest"]


def test_ring_form_constants_match_header():
    """The binding's ring-form constants are the header's NBA_IPSEC_RING_* values
    (GRAPH, PERSISTENT, PIPELINED, FREE, ROLES)."""
    import os
    import re
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    hdr = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include",
                            "nba_ipsec.h")).read()
    vals = {m.group(1): int(m.group(2)) for m in re.finditer(r"NBA_IPSEC_RING_([A-Z]+) = (\d+)", hdr)}
    for name in ("GRAPH", "PERSISTENT", "PIPELINED", "FREE", "ROLES"):
        assert getattr(nba_ipsec.Ring, name) == vals[name], name
