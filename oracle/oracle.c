/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle for the NBA IPsec
 * ESP outbound hot path (AES-128-CTR + HMAC-SHA1-96, tunnel mode).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_eurosys_kimjlmsm15_b200/) never calls it and
 * shares no code, header, table or constant generator with it.
 *
 * What it computes:
 *   PAPER.md:389 (§4.1, "Sample applications"): "IPsec encryption uses
 *   HMAC-SHA1 to authenticate the packets and AES-128CTR to encrypt them."
 *   PAPER.md:395 (§4.1): per-flow contexts are initialised once and reused
 *   "by only changing initial vector (IV) values".
 *   The paper does not define the ESP wire format; every reading below
 *   (A1..A24 of SURVEY.md §8(c), restated in DESIGN.md §3) comes from
 *   RFC 4303 (ESP), RFC 3686 (AES-CTR in ESP), RFC 2404 (HMAC-SHA1-96),
 *   RFC 2104 (HMAC), FIPS-197 (AES), FIPS 180-4 (SHA-1), RFC 1071 (checksum).
 *
 * Style: byte-oriented, no T-tables, no midstate trick, no blocking or
 * reordering; every function follows the text of the standard it cites so
 * a reader can check it by eye.  C99, libc + pthreads only.
 *
 * Pins: tests/test_oracle_*.py (FIPS-197 App. A.1/B/C.1, SP 800-38A F.5.1,
 * RFC 3686 §6, FIPS 180 examples, RFC 2202, SURVEY Appendix A worked ESP
 * example, pyca/OpenSSL random cross-checks, decap round trips, invariants).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#include "oracle.h"

/* ------------------------------------------------------------------------ */
/* FIPS-197 §4.2: multiplication in GF(2^8) modulo m(x) = x^8+x^4+x^3+x+1.   */
/* ------------------------------------------------------------------------ */

/* FIPS-197 §4.2.1: xtime(b) = b*{02}. */
static uint8_t xtime(uint8_t b)
{
    return (uint8_t)((b << 1) ^ ((b & 0x80) ? 0x1b : 0x00));
}

/* FIPS-197 §4.2.1: product by repeated xtime, one bit of b at a time. */
static uint8_t gf_mul(uint8_t a, uint8_t b)
{
    uint8_t p = 0;
    while (b) {
        if (b & 1) p ^= a;
        a = xtime(a);
        b >>= 1;
    }
    return p;
}

/* FIPS-197 §5.1.1: S-box = affine transform of the multiplicative inverse
 * in GF(2^8) ({00} maps to {00}).  The inverse is found by brute force. */
static uint8_t SBOX[256];
static int sbox_ready = 0;

static uint8_t gf_inverse(uint8_t a)
{
    if (a == 0) return 0;
    for (int b = 1; b < 256; b++)
        if (gf_mul(a, (uint8_t)b) == 1) return (uint8_t)b;
    return 0; /* unreachable: GF(2^8)* is a group */
}

static void sbox_init(void)
{
    if (sbox_ready) return;
    for (int x = 0; x < 256; x++) {
        uint8_t b = gf_inverse((uint8_t)x);
        uint8_t s = 0;
        /* b'_i = b_i ^ b_{i+4} ^ b_{i+5} ^ b_{i+6} ^ b_{i+7} ^ c_i, c = {63} */
        for (int i = 0; i < 8; i++) {
            int bit = ((b >> i) & 1) ^ ((b >> ((i + 4) % 8)) & 1) ^
                      ((b >> ((i + 5) % 8)) & 1) ^ ((b >> ((i + 6) % 8)) & 1) ^
                      ((b >> ((i + 7) % 8)) & 1) ^ ((0x63 >> i) & 1);
            s |= (uint8_t)(bit << i);
        }
        SBOX[x] = s;
    }
    sbox_ready = 1;
}

void oracle_init(void) { sbox_init(); }

uint8_t oracle_sbox(uint8_t x) { sbox_init(); return SBOX[x]; }

/* ------------------------------------------------------------------------ */
/* FIPS-197 §5.2: KeyExpansion for Nk = 4, Nr = 10 -> w[0..43] (176 bytes). */
/* w is stored as 44 words of 4 bytes each, byte order as in the standard.  */
/* ------------------------------------------------------------------------ */
void oracle_aes128_expand_key(const uint8_t key[16], uint8_t w[176])
{
    sbox_init();
    uint8_t rcon = 0x01;                       /* Rcon[i/Nk] = [x^(i/Nk-1),0,0,0] */
    memcpy(w, key, 16);
    for (int i = 4; i < 44; i++) {
        uint8_t temp[4];
        memcpy(temp, w + 4 * (i - 1), 4);
        if (i % 4 == 0) {
            /* temp = SubWord(RotWord(temp)) xor Rcon[i/Nk] */
            uint8_t t0 = temp[0];
            temp[0] = SBOX[temp[1]];
            temp[1] = SBOX[temp[2]];
            temp[2] = SBOX[temp[3]];
            temp[3] = SBOX[t0];
            temp[0] ^= rcon;
            rcon = xtime(rcon);
        }
        for (int j = 0; j < 4; j++)
            w[4 * i + j] = (uint8_t)(w[4 * (i - 4) + j] ^ temp[j]);
    }
}

/* FIPS-197 §5.1: Cipher().  state[r][c] = in[r + 4c] (§3.4). */
static void add_round_key(uint8_t s[4][4], const uint8_t *w, int round)
{
    for (int c = 0; c < 4; c++)
        for (int r = 0; r < 4; r++)
            s[r][c] ^= w[16 * round + 4 * c + r];
}

static void sub_bytes(uint8_t s[4][4])               /* §5.1.1 */
{
    for (int r = 0; r < 4; r++)
        for (int c = 0; c < 4; c++) s[r][c] = SBOX[s[r][c]];
}

static void shift_rows(uint8_t s[4][4])              /* §5.1.2 */
{
    uint8_t t[4];
    for (int r = 1; r < 4; r++) {
        for (int c = 0; c < 4; c++) t[c] = s[r][(c + r) % 4];
        for (int c = 0; c < 4; c++) s[r][c] = t[c];
    }
}

static void mix_columns(uint8_t s[4][4])             /* §5.1.3, eq. 5.6 */
{
    for (int c = 0; c < 4; c++) {
        uint8_t a0 = s[0][c], a1 = s[1][c], a2 = s[2][c], a3 = s[3][c];
        s[0][c] = (uint8_t)(gf_mul(a0, 2) ^ gf_mul(a1, 3) ^ a2 ^ a3);
        s[1][c] = (uint8_t)(a0 ^ gf_mul(a1, 2) ^ gf_mul(a2, 3) ^ a3);
        s[2][c] = (uint8_t)(a0 ^ a1 ^ gf_mul(a2, 2) ^ gf_mul(a3, 3));
        s[3][c] = (uint8_t)(gf_mul(a0, 3) ^ a1 ^ a2 ^ gf_mul(a3, 2));
    }
}

void oracle_aes128_encrypt_w(const uint8_t w[176], const uint8_t in[16], uint8_t out[16])
{
    uint8_t s[4][4];
    sbox_init();
    for (int c = 0; c < 4; c++)
        for (int r = 0; r < 4; r++) s[r][c] = in[r + 4 * c];
    add_round_key(s, w, 0);
    for (int round = 1; round < 10; round++) {
        sub_bytes(s);
        shift_rows(s);
        mix_columns(s);
        add_round_key(s, w, round);
    }
    sub_bytes(s);
    shift_rows(s);
    add_round_key(s, w, 10);
    for (int c = 0; c < 4; c++)
        for (int r = 0; r < 4; r++) out[r + 4 * c] = s[r][c];
}

void oracle_aes128_encrypt(const uint8_t key[16], const uint8_t in[16], uint8_t out[16])
{
    uint8_t w[176];
    oracle_aes128_expand_key(key, w);
    oracle_aes128_encrypt_w(w, in, out);
}

/* NIST SP 800-38A §6.5 CTR mode with the standard incrementing function of
 * Appendix B.1 applied to the last m = 32 bits of the counter block (the
 * RFC 3686 §4 block counter is exactly such a 32-bit big-endian field).
 * out = in xor (E(T1) || E(T2) || ...), truncated to len bytes. */
void oracle_ctr_xcrypt(const uint8_t key[16], const uint8_t icb[16],
                       const uint8_t *in, size_t len, uint8_t *out)
{
    uint8_t w[176], ctr[16], ks[16];
    oracle_aes128_expand_key(key, w);
    memcpy(ctr, icb, 16);
    for (size_t off = 0; off < len; off += 16) {
        oracle_aes128_encrypt_w(w, ctr, ks);
        for (size_t j = 0; j < 16 && off + j < len; j++) out[off + j] = in[off + j] ^ ks[j];
        /* [x]_32 + 1 mod 2^32 on the last four bytes, big-endian */
        for (int j = 15; j >= 12; j--) {
            ctr[j] = (uint8_t)(ctr[j] + 1);
            if (ctr[j] != 0) break;
        }
    }
}

/* ------------------------------------------------------------------------ */
/* FIPS 180-4 SHA-1: §4.1.1 functions, §4.2.1 constants, §5.1.1 padding,    */
/* §5.3.1 initial hash value, §6.1.2 hash computation.                      */
/* ------------------------------------------------------------------------ */
static uint32_t rotl32(uint32_t x, int n) { return (x << n) | (x >> (32 - n)); }

static void sha1_compress(uint32_t H[5], const uint8_t M[64])
{
    uint32_t W[80];
    for (int t = 0; t < 16; t++)
        W[t] = ((uint32_t)M[4 * t] << 24) | ((uint32_t)M[4 * t + 1] << 16) |
               ((uint32_t)M[4 * t + 2] << 8) | (uint32_t)M[4 * t + 3];
    for (int t = 16; t < 80; t++)
        W[t] = rotl32(W[t - 3] ^ W[t - 8] ^ W[t - 14] ^ W[t - 16], 1);
    uint32_t a = H[0], b = H[1], c = H[2], d = H[3], e = H[4];
    for (int t = 0; t < 80; t++) {
        uint32_t f, K;
        if (t < 20)      { f = (b & c) ^ (~b & d);           K = 0x5a827999; } /* Ch     */
        else if (t < 40) { f = b ^ c ^ d;                    K = 0x6ed9eba1; } /* Parity */
        else if (t < 60) { f = (b & c) ^ (b & d) ^ (c & d);  K = 0x8f1bbcdc; } /* Maj    */
        else             { f = b ^ c ^ d;                    K = 0xca62c1d6; } /* Parity */
        uint32_t T = rotl32(a, 5) + f + e + K + W[t];
        e = d; d = c; c = rotl32(b, 30); b = a; a = T;
    }
    H[0] += a; H[1] += b; H[2] += c; H[3] += d; H[4] += e;
}

void oracle_sha1(const uint8_t *msg, size_t len, uint8_t out[20])
{
    uint32_t H[5] = {0x67452301, 0xefcdab89, 0x98badcfe, 0x10325476, 0xc3d2e1f0};
    /* §5.1.1: append 1 bit, k zero bits, 64-bit big-endian bit length. */
    size_t padded = ((len + 8) / 64 + 1) * 64;
    uint8_t *buf = (uint8_t *)calloc(padded, 1);
    if (!buf) { memset(out, 0, 20); return; }
    if (len) memcpy(buf, msg, len);
    buf[len] = 0x80;
    uint64_t bits = (uint64_t)len * 8u;
    for (int j = 0; j < 8; j++) buf[padded - 1 - j] = (uint8_t)(bits >> (8 * j));
    for (size_t off = 0; off < padded; off += 64) sha1_compress(H, buf + off);
    free(buf);
    for (int i = 0; i < 5; i++) {
        out[4 * i] = (uint8_t)(H[i] >> 24);
        out[4 * i + 1] = (uint8_t)(H[i] >> 16);
        out[4 * i + 2] = (uint8_t)(H[i] >> 8);
        out[4 * i + 3] = (uint8_t)H[i];
    }
}

/* RFC 2104 §2: HMAC(K, text) = H(K0 xor opad, H(K0 xor ipad, text)),
 * K0 = K zero-padded to B = 64 bytes (or H(K) padded, if |K| > B). */
void oracle_hmac_sha1(const uint8_t *key, size_t klen, const uint8_t *msg, size_t mlen,
                      uint8_t out[20])
{
    uint8_t K0[64];
    memset(K0, 0, 64);
    if (klen > 64) oracle_sha1(key, klen, K0);
    else if (klen) memcpy(K0, key, klen);

    uint8_t *inner = (uint8_t *)malloc(64 + mlen);
    uint8_t outer[64 + 20];
    if (!inner) { memset(out, 0, 20); return; }
    for (int i = 0; i < 64; i++) inner[i] = K0[i] ^ 0x36;
    if (mlen) memcpy(inner + 64, msg, mlen);
    uint8_t ih[20];
    oracle_sha1(inner, 64 + mlen, ih);
    free(inner);
    for (int i = 0; i < 64; i++) outer[i] = K0[i] ^ 0x5c;
    memcpy(outer + 64, ih, 20);
    oracle_sha1(outer, 84, out);
}

/* RFC 1071 §4.1: ones'-complement of the ones'-complement sum of 16-bit
 * big-endian words. Returned in host order; store big-endian. */
uint16_t oracle_ipv4_checksum(const uint8_t *hdr, size_t len)
{
    uint32_t sum = 0;
    for (size_t i = 0; i + 1 < len; i += 2) sum += ((uint32_t)hdr[i] << 8) | hdr[i + 1];
    if (len & 1) sum += (uint32_t)hdr[len - 1] << 8;
    while (sum >> 16) sum = (sum & 0xffff) + (sum >> 16);
    return (uint16_t)~sum;
}

/* ------------------------------------------------------------------------ */
/* ESP outbound, tunnel mode: SURVEY.md §8(c) steps 1..8 / DESIGN.md §3.    */
/* ------------------------------------------------------------------------ */
static void put_be32(uint8_t *p, uint32_t v)
{
    p[0] = (uint8_t)(v >> 24); p[1] = (uint8_t)(v >> 16); p[2] = (uint8_t)(v >> 8); p[3] = (uint8_t)v;
}

/* Encapsulate one packet P (D bytes) with sequence number q under SA sa.
 * Writes O||H||E||ICV (48+C bytes) to out, returns 48+C. */
uint32_t oracle_esp_encap(const oracle_sa *sa, uint32_t q, const uint8_t *P, uint32_t D, uint8_t *out)
{
    /* step 3: IV = BE64(q) (RFC 3686 §3.1 allows any unique IV; A6) */
    uint8_t IV[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    put_be32(IV + 4, q);

    /* step 4: T = P || 01 02 .. p || p || 04, p = (-(D+2)) mod 4 (A9, A10) */
    uint32_t p = (4u - ((D + 2u) % 4u)) % 4u;
    uint32_t C = D + p + 2u;
    uint8_t *T = (uint8_t *)malloc(C);
    if (!T) return 0;
    memcpy(T, P, D);
    for (uint32_t j = 1; j <= p; j++) T[D + j - 1] = (uint8_t)j;
    T[D + p] = (uint8_t)p;        /* Pad Length   (RFC 4303 §2.5) */
    T[D + p + 1] = 4;             /* Next Header: IPv4 (RFC 4303 §2.6; tunnel mode) */

    /* step 5: E = T xor keystream, counter block nonce || IV || BE32(1..) (RFC 3686 §4) */
    uint8_t icb[16];
    memcpy(icb, sa->ctr_nonce, 4);
    memcpy(icb + 4, IV, 8);
    put_be32(icb + 12, 1);
    uint8_t *E = out + 20 + 16;
    oracle_ctr_xcrypt(sa->aes_key, icb, T, C, E);
    free(T);

    /* step 6: H = BE32(spi) || BE32(q) || IV ; ICV = HMAC-SHA1(H || E)[0:12] */
    uint8_t *H = out + 20;
    put_be32(H, sa->spi);
    put_be32(H + 4, q);
    memcpy(H + 8, IV, 8);
    uint8_t mac[20];
    oracle_hmac_sha1(sa->hmac_key, 20, H, 16 + C, mac);   /* covers H and E (§3.3.4) */
    memcpy(out + 20 + 16 + C, mac, 12);                    /* RFC 2404 §2: first 96 bits */

    /* step 7: outer IPv4 header (A13) */
    uint8_t *O = out;
    uint32_t tot = 48u + C;
    O[0] = 0x45;
    O[1] = P[1];                  /* TOS copied from the inner header */
    O[2] = (uint8_t)(tot >> 8); O[3] = (uint8_t)tot;
    O[4] = 0; O[5] = 0;           /* identification 0 */
    O[6] = 0x40; O[7] = 0x00;     /* DF, fragment offset 0 */
    O[8] = 64;                    /* TTL */
    O[9] = 50;                    /* protocol ESP */
    O[10] = 0; O[11] = 0;
    put_be32(O + 12, sa->tunnel_src);
    put_be32(O + 16, sa->tunnel_dst);
    uint16_t cs = oracle_ipv4_checksum(O, 20);
    O[10] = (uint8_t)(cs >> 8); O[11] = (uint8_t)cs;
    return tot;
}

/* Sequential batch loop, packets in index order.
 * sas[].seq is updated in place; counters are accumulated into *ctr. */
void oracle_process_batch(oracle_sa *sas, uint32_t n_sa,
                          const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                          const uint32_t *sa_idx, uint8_t *out_buf, const uint32_t *out_off,
                          uint16_t *out_len, uint32_t n, oracle_counters *ctr)
{
    sbox_init();
    for (uint32_t i = 0; i < n; i++) {
        uint32_t s = sa_idx[i];
        uint32_t D = in_len[i];
        /* step 1: invalid SA or length -> drop, no seq consumed (A15) */
        if (s >= n_sa || D < ORACLE_MIN_DATAGRAM || D > ORACLE_MAX_DATAGRAM) {
            out_len[i] = 0;
            ctr->pkts_dropped++;
            continue;
        }
        /* step 2: the counter must not cycle (RFC 4303 §3.3.3) */
        if (sas[s].seq == 0xffffffffu) {
            out_len[i] = 0;
            ctr->pkts_dropped++;
            continue;
        }
        sas[s].seq += 1;
        uint32_t q = sas[s].seq;
        uint32_t L = oracle_esp_encap(&sas[s], q, in_buf + in_off[i], D, out_buf + out_off[i]);
        out_len[i] = (uint16_t)L;
        ctr->pkts_ok++;
        ctr->bytes_in += D;
        ctr->bytes_out += L;
    }
    if (n) ctr->batches++;
}

/* Parallel variant used only to time the oracle on many host cores:
 * thread t owns SAs with s mod T == t and scans all packets in index order,
 * so per-SA order and every output byte are identical to the sequential
 * loop (tests/test_oracle_esp.py checks that identity). */
typedef struct {
    oracle_sa *sas; uint32_t n_sa;
    const uint8_t *in_buf; const uint32_t *in_off; const uint16_t *in_len; const uint32_t *sa_idx;
    uint8_t *out_buf; const uint32_t *out_off; uint16_t *out_len; uint32_t n;
    uint32_t t, T;
    oracle_counters ctr;
} mt_arg;

static void *mt_worker(void *argp)
{
    mt_arg *a = (mt_arg *)argp;
    for (uint32_t i = 0; i < a->n; i++) {
        uint32_t s = a->sa_idx[i];
        uint32_t D = a->in_len[i];
        uint32_t owner = (s < a->n_sa) ? (s % a->T) : 0;   /* bad-SA drops: thread 0 */
        if (owner != a->t) continue;
        if (s >= a->n_sa || D < ORACLE_MIN_DATAGRAM || D > ORACLE_MAX_DATAGRAM ||
            a->sas[s].seq == 0xffffffffu) {
            a->out_len[i] = 0;
            a->ctr.pkts_dropped++;
            continue;
        }
        a->sas[s].seq += 1;
        uint32_t L = oracle_esp_encap(&a->sas[s], a->sas[s].seq, a->in_buf + a->in_off[i], D,
                                      a->out_buf + a->out_off[i]);
        a->out_len[i] = (uint16_t)L;
        a->ctr.pkts_ok++;
        a->ctr.bytes_in += D;
        a->ctr.bytes_out += L;
    }
    return NULL;
}

int oracle_process_batch_mt(oracle_sa *sas, uint32_t n_sa,
                            const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                            const uint32_t *sa_idx, uint8_t *out_buf, const uint32_t *out_off,
                            uint16_t *out_len, uint32_t n, oracle_counters *ctr, int n_threads)
{
    sbox_init();
    if (n_threads < 1) n_threads = 1;
    mt_arg *args = (mt_arg *)calloc((size_t)n_threads, sizeof(mt_arg));
    pthread_t *th = (pthread_t *)calloc((size_t)n_threads, sizeof(pthread_t));
    if (!args || !th) { free(args); free(th); return -1; }
    for (int t = 0; t < n_threads; t++) {
        mt_arg *a = &args[t];
        a->sas = sas; a->n_sa = n_sa; a->in_buf = in_buf; a->in_off = in_off; a->in_len = in_len;
        a->sa_idx = sa_idx; a->out_buf = out_buf; a->out_off = out_off; a->out_len = out_len;
        a->n = n; a->t = (uint32_t)t; a->T = (uint32_t)n_threads;
        if (t > 0) pthread_create(&th[t], NULL, mt_worker, a);
    }
    mt_worker(&args[0]);
    for (int t = 1; t < n_threads; t++) pthread_join(th[t], NULL);
    for (int t = 0; t < n_threads; t++) {
        ctr->pkts_ok += args[t].ctr.pkts_ok;
        ctr->pkts_dropped += args[t].ctr.pkts_dropped;
        ctr->bytes_in += args[t].ctr.bytes_in;
        ctr->bytes_out += args[t].ctr.bytes_out;
    }
    if (n) ctr->batches++;
    free(args);
    free(th);
    return 0;
}

/* ESP inbound for tests (SURVEY §8(c) "Decap"): parse the outer header,
 * check its checksum, verify the ICV, decrypt, check the trailer, return P.
 * Returns 0 on success, a negative ORACLE_E* code otherwise. */
int oracle_decap(const oracle_sa *sa, const uint8_t *pkt, uint32_t len,
                 uint8_t *inner, uint32_t *inner_len, uint32_t *seq_out)
{
    if (len < 20 + 16 + 4 + 12) return ORACLE_EFORMAT;
    if (pkt[0] != 0x45 || pkt[9] != 50) return ORACLE_EFORMAT;
    if ((((uint32_t)pkt[2] << 8) | pkt[3]) != len) return ORACLE_EFORMAT;
    if (oracle_ipv4_checksum(pkt, 20) != 0) return ORACLE_ECSUM;   /* folds to 0xffff */
    const uint8_t *H = pkt + 20;
    uint32_t C = len - 48;
    if (C % 4 != 0) return ORACLE_EFORMAT;
    uint32_t spi = ((uint32_t)H[0] << 24) | ((uint32_t)H[1] << 16) | ((uint32_t)H[2] << 8) | H[3];
    if (spi != sa->spi) return ORACLE_EFORMAT;
    uint8_t mac[20];
    oracle_hmac_sha1(sa->hmac_key, 20, H, 16 + C, mac);
    uint8_t diff = 0;
    for (int j = 0; j < 12; j++) diff |= (uint8_t)(mac[j] ^ H[16 + C + j]);
    if (diff) return ORACLE_EICV;
    uint8_t icb[16];
    memcpy(icb, sa->ctr_nonce, 4);
    memcpy(icb + 4, H + 8, 8);
    put_be32(icb + 12, 1);
    uint8_t *T = (uint8_t *)malloc(C);
    if (!T) return ORACLE_EFORMAT;
    oracle_ctr_xcrypt(sa->aes_key, icb, H + 16, C, T);
    uint32_t p = T[C - 2];
    int rc = 0;
    if (T[C - 1] != 4 || p > 3 || p + 2 > C) rc = ORACLE_ETRAILER;
    for (uint32_t j = 1; rc == 0 && j <= p; j++)
        if (T[C - 2 - p + j - 1] != (uint8_t)j) rc = ORACLE_ETRAILER;
    if (rc == 0) {
        *inner_len = C - 2 - p;
        memcpy(inner, T, *inner_len);
        if (seq_out)
            *seq_out = ((uint32_t)H[4] << 24) | ((uint32_t)H[5] << 16) | ((uint32_t)H[6] << 8) | H[7];
    }
    free(T);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* ESP inbound, sequential.  RFC 4303 §3.4 in its order:    */
/* §3.4.1 no fragments, §3.4.2 SA (caller's sa_idx, SPI must match),         */
/* §3.4.3 sequence number / anti-replay check, §3.4.4.1 ICV check, then the  */
/* receive window update ("only if the integrity verification succeeds"),   */
/* §3.4.4.2 decryption, §2.4 / §2.6 trailer checks, output of the inner      */
/* datagram.  Readings B1..B9 are listed in DESIGN.md.                       */
/* ------------------------------------------------------------------------ */

/* B6: the window starts at the SA's `seq` with everything at or below it
 * counted as received (a resumed SA); seq = 0 gives an empty window. */
void oracle_replay_init(const oracle_sa *sa, oracle_replay *w)
{
    w->top = sa->seq;
    w->pad_ = 0;
    w->bitmap = sa->seq ? ~(uint64_t)0 : 0;
}

/* RFC 4303 §3.4.3: right edge `top` = highest authenticated number; bit d of
 * the bitmap records number top - d (d < 64).  Zero is never sent (§3.3.3). */
static int replay_check(const oracle_replay *w, uint32_t q)
{
    if (q == 0) return 0;
    if (q > w->top) return 1;                       /* right of the window: new */
    uint32_t d = w->top - q;
    if (d >= ORACLE_REPLAY_WINDOW) return 0;        /* left of the window: too old */
    return ((w->bitmap >> d) & 1u) ? 0 : 1;         /* inside: not seen before */
}

static void replay_update(oracle_replay *w, uint32_t q)
{
    if (q > w->top) {                               /* slide the window right */
        uint32_t shift = q - w->top;
        w->bitmap = shift >= ORACLE_REPLAY_WINDOW ? 0 : (w->bitmap << shift);
        w->bitmap |= 1u;
        w->top = q;
    } else {
        w->bitmap |= (uint64_t)1 << (w->top - q);
    }
}

static uint32_t be32_at(const uint8_t *p)
{
    return ((uint32_t)p[0] << 24) | ((uint32_t)p[1] << 16) | ((uint32_t)p[2] << 8) | p[3];
}

/* One packet; returns its ORACLE_IN_* status and the inner length in *D_out. */
static int inbound_one(const oracle_sa *sa, oracle_replay *w, const uint8_t *pkt, uint32_t L,
                       uint8_t *out, uint32_t *D_out)
{
    /* B2: outer IPv4 without options, not a fragment (§3.4.1), protocol ESP,
     * total length = the caller's length, valid header checksum (RFC 1071) */
    if (L < 48u + 24u || L > 48u + 1504u || (L - 48u) % 4u != 0) return ORACLE_IN_DROP_FORMAT;
    if (pkt[0] != 0x45 || pkt[9] != 50) return ORACLE_IN_DROP_FORMAT;
    if ((((uint32_t)pkt[2] << 8) | pkt[3]) != L) return ORACLE_IN_DROP_FORMAT;
    if (((((uint32_t)pkt[6] << 8) | pkt[7]) & 0x3fffu) != 0) return ORACLE_IN_DROP_FORMAT;
    if (oracle_ipv4_checksum(pkt, 20) != 0) return ORACLE_IN_DROP_FORMAT;
    const uint8_t *H = pkt + 20;                     /* SPI || seq || IV */
    if (be32_at(H) != sa->spi) return ORACLE_IN_DROP_FORMAT;     /* §3.4.2 */
    const uint32_t C = L - 48u;
    const uint32_t q = be32_at(H + 4);

    /* §3.4.3: sequence number check before the ICV */
    if (!replay_check(w, q)) return ORACLE_IN_DROP_REPLAY;

    /* §3.4.4.1: ICV = HMAC-SHA1(H || E)[0:12], compared without early exit */
    uint8_t mac[20];
    oracle_hmac_sha1(sa->hmac_key, 20, H, 16u + C, mac);
    uint8_t diff = 0;
    for (int j = 0; j < 12; j++) diff |= (uint8_t)(mac[j] ^ H[16u + C + (uint32_t)j]);
    if (diff) return ORACLE_IN_DROP_AUTH;

    /* §3.4.3: the window advances only for authenticated packets */
    replay_update(w, q);

    /* §3.4.4.2: T = E xor keystream; counter block nonce || IV(from packet) || BE32(1..) */
    uint8_t icb[16];
    memcpy(icb, sa->ctr_nonce, 4);
    memcpy(icb + 4, H + 8, 8);
    put_be32(icb + 12, 1);
    uint8_t *T = (uint8_t *)malloc(C);
    if (!T) return ORACLE_IN_DROP_FORMAT;
    oracle_ctr_xcrypt(sa->aes_key, icb, H + 16, C, T);

    /* B4: next header 4 (tunnel mode), pad bytes 1..p (§2.4), D >= 20 */
    int rc = ORACLE_IN_OK;
    const uint32_t p = T[C - 2];
    if (T[C - 1] != 4 || p + 2u + ORACLE_MIN_DATAGRAM > C) rc = ORACLE_IN_DROP_TRAILER;
    const uint32_t D = C - 2u - p;
    for (uint32_t j = 1; rc == ORACLE_IN_OK && j <= p; j++)
        if (T[D + j - 1] != (uint8_t)j) rc = ORACLE_IN_DROP_TRAILER;
    if (rc == ORACLE_IN_OK) {
        memcpy(out, T, D);
        *D_out = D;
    }
    free(T);
    return rc;
}

void oracle_process_inbound(const oracle_sa *sas, oracle_replay *win, uint32_t n_sa,
                            const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                            const uint32_t *sa_idx, uint8_t *out_buf, const uint32_t *out_off,
                            uint16_t *out_len, uint8_t *status, uint32_t n,
                            oracle_in_counters *ctr)
{
    sbox_init();
    for (uint32_t i = 0; i < n; i++) {
        const uint32_t s = sa_idx[i];
        uint32_t D = 0;
        int rc = s < n_sa ? inbound_one(&sas[s], &win[s], in_buf + in_off[i], in_len[i],
                                        out_buf + out_off[i], &D)
                          : ORACLE_IN_DROP_SA;
        status[i] = (uint8_t)rc;
        out_len[i] = rc == ORACLE_IN_OK ? (uint16_t)D : 0;
        switch (rc) {
        case ORACLE_IN_OK:
            ctr->pkts_ok++;
            ctr->bytes_in += in_len[i];
            ctr->bytes_out += D;
            break;
        case ORACLE_IN_DROP_SA: ctr->drop_sa++; break;
        case ORACLE_IN_DROP_FORMAT: ctr->drop_format++; break;
        case ORACLE_IN_DROP_REPLAY: ctr->drop_replay++; break;
        case ORACLE_IN_DROP_AUTH: ctr->drop_auth++; break;
        default: ctr->drop_trailer++; break;
        }
    }
    if (n) ctr->batches++;
}

/* ------------------------------------------------------------------------ */
/* Flow -> SA lookup.  PAPER.md:395 keeps one crypto      */
/* context per flow, initialised at startup; the lookup is an exact match   */
/* on the inner IPv4 5-tuple (readings F1..F4 in DESIGN.md): plain parsing  */
/* of the header and a binary search over the sorted flow list.             */
/* ------------------------------------------------------------------------ */
static int flow_cmp(const oracle_flow *a, const oracle_flow *b)
{
    if (a->src != b->src) return a->src < b->src ? -1 : 1;
    if (a->dst != b->dst) return a->dst < b->dst ? -1 : 1;
    if (a->proto != b->proto) return a->proto < b->proto ? -1 : 1;
    if (a->sport != b->sport) return a->sport < b->sport ? -1 : 1;
    if (a->dport != b->dport) return a->dport < b->dport ? -1 : 1;
    return 0;
}

static int flow_qsort_cmp(const void *a, const void *b)
{
    return flow_cmp((const oracle_flow *)a, (const oracle_flow *)b);
}

int oracle_flow_table_prepare(oracle_flow *flows, uint32_t n_flows)
{
    qsort(flows, n_flows, sizeof(oracle_flow), flow_qsort_cmp);
    for (uint32_t k = 1; k < n_flows; k++)
        if (flow_cmp(&flows[k - 1], &flows[k]) == 0) return -1;
    return 0;
}

/* F1/F2: the key of one inner datagram; returns 0 if it has none. */
static int flow_key(const uint8_t *P, uint32_t D, oracle_flow *k)
{
    if (D < 20) return 0;
    uint32_t ihl = P[0] & 0x0fu;
    if ((P[0] >> 4) != 4 || ihl < 5 || D < 4u * ihl) return 0;
    memset(k, 0, sizeof(*k));
    k->src = be32_at(P + 12);
    k->dst = be32_at(P + 16);
    k->proto = P[9];
    uint32_t frag_off = (((uint32_t)P[6] << 8) | P[7]) & 0x1fffu;
    if ((k->proto == 6 || k->proto == 17) && frag_off == 0 && D >= 4u * ihl + 4u) {
        k->sport = (uint16_t)(((uint32_t)P[4 * ihl] << 8) | P[4 * ihl + 1]);
        k->dport = (uint16_t)(((uint32_t)P[4 * ihl + 2] << 8) | P[4 * ihl + 3]);
    }
    return 1;
}

void oracle_flow_lookup(const oracle_flow *sorted_flows, uint32_t n_flows,
                        const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                        uint32_t n, uint32_t *sa_idx)
{
    for (uint32_t i = 0; i < n; i++) {
        oracle_flow k;
        sa_idx[i] = ORACLE_NO_SA;
        if (!flow_key(in_buf + in_off[i], in_len[i], &k)) continue;
        const oracle_flow *hit = (const oracle_flow *)bsearch(&k, sorted_flows, n_flows,
                                                              sizeof(oracle_flow), flow_qsort_cmp);
        if (hit) sa_idx[i] = hit->sa;
    }
}
