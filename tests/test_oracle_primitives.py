"""Pins for the oracle's primitives (tier T1): FIPS-197, SP 800-38A, RFC 3686,
FIPS 180, RFC 2202, plus random cross-checks against OpenSSL (pyca/hashlib)."""
import hashlib
import hmac

import numpy as np
import pytest
from cryptography.hazmat.primitives.ciphers import Cipher, algorithms, modes

import oracle
from golden import load, msg_of

AES = load("aes_vectors.txt")
SHA = load("sha1_hmac_vectors.txt")


def test_sbox_spot_values_and_permutation():
    # FIPS-197 §5.1.1 / Fig. 7: S(00)=63, S(53)=ED; Sbox is a bijection.
    assert oracle.sbox(0x00) == 0x63
    assert oracle.sbox(0x53) == 0xED
    assert oracle.sbox(0x01) == 0x7C and oracle.sbox(0xFF) == 0x16
    assert sorted(oracle.sbox(x) for x in range(256)) == list(range(256))
    # no fixed points and no "opposite" fixed points (design property, FIPS-197 §5.1.1 note)
    assert all(oracle.sbox(x) != x and oracle.sbox(x) != (x ^ 0xFF) for x in range(256))


def test_key_expansion_fips197_a1():
    r = AES["fips197_a1"]
    w = oracle.aes128_expand_key(bytes.fromhex(r["key"]))
    assert w[:16] == bytes.fromhex(r["key"])
    assert w[16:32].hex() == r["w4_7"]
    assert w[160:176].hex() == r["w40_43"]


@pytest.mark.parametrize("name", ["fips197_c1", "fips197_b"])
def test_aes_block_known_answer(name):
    r = AES[name]
    assert oracle.aes128_encrypt(bytes.fromhex(r["key"]), bytes.fromhex(r["plaintext"])).hex() \
        == r["ciphertext"]


def test_ctr_sp800_38a_f51():
    r = AES["sp800_38a_f51"]
    out = oracle.ctr_xcrypt(bytes.fromhex(r["key"]), bytes.fromhex(r["icb"]),
                            bytes.fromhex(r["plaintext"]))
    assert out.hex() == r["ciphertext"]


@pytest.mark.parametrize("name", ["rfc3686_1", "rfc3686_2", "rfc3686_3"])
def test_ctr_rfc3686(name):
    r = AES[name]
    icb = bytes.fromhex(r["nonce"] + r["iv"]) + b"\x00\x00\x00\x01"
    out = oracle.ctr_xcrypt(bytes.fromhex(r["key"]), icb, bytes.fromhex(r["plaintext"]))
    assert out.hex() == r["ciphertext"]
    # CTR is an involution
    assert oracle.ctr_xcrypt(bytes.fromhex(r["key"]), icb, out).hex() == r["plaintext"]


def test_aes_random_vs_openssl():
    rng = np.random.default_rng(1)
    for _ in range(300):
        k = rng.integers(0, 256, 16, dtype=np.uint8).tobytes()
        b = rng.integers(0, 256, 16, dtype=np.uint8).tobytes()
        e = Cipher(algorithms.AES(k), modes.ECB()).encryptor()
        assert oracle.aes128_encrypt(k, b) == e.update(b) + e.finalize()


def test_ctr_random_vs_openssl_including_counter_carry():
    rng = np.random.default_rng(2)
    for i in range(100):
        k = rng.integers(0, 256, 16, dtype=np.uint8).tobytes()
        icb = bytearray(rng.integers(0, 256, 16, dtype=np.uint8).tobytes())
        if i % 4 == 0:
            icb[12:16] = b"\x00\x00\xff\xfe"        # carry across bytes inside the 32-bit field
        data = rng.integers(0, 256, int(rng.integers(0, 200)), dtype=np.uint8).tobytes()
        e = Cipher(algorithms.AES(k), modes.CTR(bytes(icb))).encryptor()
        assert oracle.ctr_xcrypt(k, bytes(icb), data) == e.update(data) + e.finalize()


@pytest.mark.parametrize("name", ["sha1_abc", "sha1_448", "sha1_million_a", "sha1_empty"])
def test_sha1_fips180(name):
    r = SHA[name]
    assert oracle.sha1(msg_of(r)).hex() == r["digest"]


@pytest.mark.parametrize("name", [f"rfc2202_{i}" for i in range(1, 8)])
def test_hmac_rfc2202(name):
    r = SHA[name]
    d = oracle.hmac_sha1(bytes.fromhex(r["key"]), msg_of(r))
    assert d.hex() == r["digest"]
    if "digest96" in r:
        assert d[:12].hex() == r["digest96"]


def test_sha1_hmac_random_lengths_vs_openssl():
    # every length around the 55/56/64-byte padding boundaries and beyond
    rng = np.random.default_rng(3)
    for n in list(range(0, 140)) + [183, 184, 191, 192, 1000, 1536, 1600]:
        m = rng.integers(0, 256, n, dtype=np.uint8).tobytes()
        assert oracle.sha1(m) == hashlib.sha1(m).digest()
        k = rng.integers(0, 256, int(rng.integers(0, 100)), dtype=np.uint8).tobytes()
        assert oracle.hmac_sha1(k, m) == hmac.new(k, m, hashlib.sha1).digest()


def test_ipv4_checksum_rfc1071():
    # A textbook header (RFC 1071-style example; checksum b861) and the fold-to-zero property.
    h = bytes.fromhex("450000730000400040110000c0a80001c0a800c7")
    assert oracle.ipv4_checksum(h) == 0xB861
    h2 = h[:10] + bytes.fromhex("b861") + h[12:]
    assert oracle.ipv4_checksum(h2) == 0
