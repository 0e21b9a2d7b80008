/*
 * oracle.h -- CPU oracle for the NBA IPsec ESP hot path.  TEST INFRASTRUCTURE
 * ONLY (see oracle.c header).  Independent of include/nba_ipsec.h: nothing
 * here is shared with the CUDA library and neither side includes the other.
 */
#ifndef NBA_ORACLE_H
#define NBA_ORACLE_H
#include <stddef.h>
#include <stdint.h>

#define ORACLE_MIN_DATAGRAM 20u    /* A15: smallest IPv4 datagram */
#define ORACLE_MAX_DATAGRAM 1500u  /* A15: paper's largest size */

#define ORACLE_EFORMAT  -1
#define ORACLE_ECSUM    -2
#define ORACLE_EICV     -3
#define ORACLE_ETRAILER -4

typedef struct {
    uint32_t spi;
    uint32_t tunnel_src, tunnel_dst;
    uint8_t  aes_key[16];
    uint8_t  ctr_nonce[4];
    uint8_t  hmac_key[20];
    uint32_t seq;                 /* last sequence number used */
} oracle_sa;

typedef struct { uint64_t pkts_ok, pkts_dropped, bytes_in, bytes_out, batches; } oracle_counters;

void     oracle_init(void);
uint8_t  oracle_sbox(uint8_t x);
void     oracle_aes128_expand_key(const uint8_t key[16], uint8_t w[176]);
void     oracle_aes128_encrypt_w(const uint8_t w[176], const uint8_t in[16], uint8_t out[16]);
void     oracle_aes128_encrypt(const uint8_t key[16], const uint8_t in[16], uint8_t out[16]);
void     oracle_ctr_xcrypt(const uint8_t key[16], const uint8_t icb[16], const uint8_t *in,
                           size_t len, uint8_t *out);
void     oracle_sha1(const uint8_t *msg, size_t len, uint8_t out[20]);
void     oracle_hmac_sha1(const uint8_t *key, size_t klen, const uint8_t *msg, size_t mlen,
                          uint8_t out[20]);
uint16_t oracle_ipv4_checksum(const uint8_t *hdr, size_t len);
uint32_t oracle_esp_encap(const oracle_sa *sa, uint32_t q, const uint8_t *P, uint32_t D,
                          uint8_t *out);
void     oracle_process_batch(oracle_sa *sas, uint32_t n_sa, const uint8_t *in_buf,
                              const uint32_t *in_off, const uint16_t *in_len,
                              const uint32_t *sa_idx, uint8_t *out_buf, const uint32_t *out_off,
                              uint16_t *out_len, uint32_t n, oracle_counters *ctr);
int      oracle_process_batch_mt(oracle_sa *sas, uint32_t n_sa, const uint8_t *in_buf,
                                 const uint32_t *in_off, const uint16_t *in_len,
                                 const uint32_t *sa_idx, uint8_t *out_buf,
                                 const uint32_t *out_off, uint16_t *out_len, uint32_t n,
                                 oracle_counters *ctr, int n_threads);
int      oracle_decap(const oracle_sa *sa, const uint8_t *pkt, uint32_t len, uint8_t *inner,
                      uint32_t *inner_len, uint32_t *seq_out);

/* ---- ESP inbound (readings B1..B9) ------------ */
#define ORACLE_IN_OK           0
#define ORACLE_IN_DROP_SA      1   /* sa_idx >= n_sa                              */
#define ORACLE_IN_DROP_FORMAT  2   /* outer header / length / SPI                 */
#define ORACLE_IN_DROP_REPLAY  3   /* RFC 4303 §3.4.3 sequence number check       */
#define ORACLE_IN_DROP_AUTH    4   /* RFC 4303 §3.4.4.1 ICV mismatch              */
#define ORACLE_IN_DROP_TRAILER 5   /* pad contents / pad length / next header     */
#define ORACLE_REPLAY_WINDOW  64u  /* RFC 4303 §3.4.3: 64 SHOULD be the default   */

typedef struct { uint32_t top; uint32_t pad_; uint64_t bitmap; } oracle_replay;
typedef struct {
    uint64_t pkts_ok, drop_sa, drop_format, drop_replay, drop_auth, drop_trailer;
    uint64_t bytes_in, bytes_out, batches;
} oracle_in_counters;

void     oracle_replay_init(const oracle_sa *sa, oracle_replay *w);
void     oracle_process_inbound(const oracle_sa *sas, oracle_replay *win, uint32_t n_sa,
                                const uint8_t *in_buf, const uint32_t *in_off,
                                const uint16_t *in_len, const uint32_t *sa_idx, uint8_t *out_buf,
                                const uint32_t *out_off, uint16_t *out_len, uint8_t *status,
                                uint32_t n, oracle_in_counters *ctr);

/* ---- flow -> SA lookup (readings F1..F4) -------- */
#define ORACLE_NO_SA 0xffffffffu
typedef struct {
    uint32_t src, dst;        /* IPv4 addresses, host order */
    uint16_t sport, dport;    /* 0 when the protocol has no ports (F2) */
    uint8_t  proto;
    uint8_t  pad_[3];
    uint32_t sa;              /* SA index of the flow */
} oracle_flow;

/* Sorts `flows` in place (the lookup is a binary search); returns -1 if two
 * flows have the same key. */
int      oracle_flow_table_prepare(oracle_flow *flows, uint32_t n_flows);
void     oracle_flow_lookup(const oracle_flow *sorted_flows, uint32_t n_flows,
                            const uint8_t *in_buf, const uint32_t *in_off, const uint16_t *in_len,
                            uint32_t n, uint32_t *sa_idx);
#endif
