"""GPU parity (tiers T5-T7, T9): the CUDA path through the C ABI against the
oracle, element by element over the WHOLE output pool (so bytes outside each
slot's [0, out_len) must stay untouched), plus out_len, final SA sequence
numbers and device counters.  Bit-exact: this is integer/byte work."""
import numpy as np
import pytest

from golden import load
from harness import assert_same, gpu_run, oracle_run
from paper_conf_eurosys_kimjlmsm15_b200 import gen

pytestmark = pytest.mark.gpu

PIPES = [0, 1]   # NBA_IPSEC_PIPE_FUSED, NBA_IPSEC_PIPE_UNFUSED


@pytest.mark.parametrize("pipe", PIPES)
def test_config1_64x64B_1sa(pipe):
    c = gen.CONFIGS[1]
    p = gen.make_sas(c["n_sa"], cfg_id=1)
    bs = [gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=1, batch=k) for k in range(3)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("pipe", PIPES)
@pytest.mark.parametrize("cfg", [2, 3, 4])
def test_full_size_configs(cfg, pipe):
    """BASELINE.json configs[1..3] at full size (65,536 packets, 1024 SAs),
    three consecutive batches so sequence state carries over."""
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    bs = [gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg, batch=k) for k in range(3)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("pipe", PIPES)
def test_worked_example(pipe):
    ex = load("esp_worked_example.txt")
    r = ex["sa"]
    p = gen.SAParams(
        spi=np.array([int(r["spi"], 16)], np.uint32),
        tunnel_src=np.array([int(r["tunnel_src"], 16)], np.uint32),
        tunnel_dst=np.array([int(r["tunnel_dst"], 16)], np.uint32),
        aes_key=np.frombuffer(bytes.fromhex(r["aes_key"]), np.uint8)[None].copy(),
        ctr_nonce=np.frombuffer(bytes.fromhex(r["nonce"]), np.uint8)[None].copy(),
        hmac_key=np.frombuffer(bytes.fromhex(r["hmac_key"]), np.uint8)[None].copy(),
        seq=np.zeros(1, np.uint32))
    pk = [bytes.fromhex(ex["pkt1"]["inner"]), bytes.fromhex(ex["pkt2"]["inner"])]
    b = gen.make_batch(2, 64, 1, in_len_override=[len(x) for x in pk], sa_idx_override=[0, 0])
    for i, x in enumerate(pk):
        b.in_buf[b.in_off[i]:b.in_off[i] + len(x)] = np.frombuffer(x, np.uint8)
    (res, seq, ctr) = gpu_run(p, [b], pipeline=pipe)
    out, ol = res[0]
    for i, name in enumerate(["pkt1", "pkt2"]):
        exp = bytes.fromhex(ex[name]["output"])
        assert int(ol[i]) == len(exp)
        assert out[b.out_off[i]:b.out_off[i] + len(exp)].tobytes() == exp
    assert seq.tolist() == [2]


@pytest.mark.parametrize("pipe", PIPES)
@pytest.mark.parametrize("n,size,n_sa,loc", [
    (5000, "imix", 37, 1),        # several tiles + ragged tail
    (3001, 1514, 5, 1),
    (4099, 64, 1, 1),             # one SA: ranks chain across tiles
    (2500, "imix", 1024, 16),     # flow locality: runs of 16 packets per SA
    (1, 1514, 3, 1),
    (33, 594, 2, 1),
])
def test_medium_shapes(n, size, n_sa, loc, pipe):
    p = gen.make_sas(n_sa, cfg_id=50)
    bs = [gen.make_batch(n, size, n_sa, cfg_id=50, batch=k, locality=loc) for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("pipe", PIPES)
def test_random_lengths_and_invalid_packets(pipe):
    """Every D in [0, 1600) with random SA indices, some >= n_sa: drops, pads 0..3."""
    rng = np.random.default_rng(7)
    n, n_sa = 6000, 11
    D = rng.integers(0, 1600, n)
    D[:8] = [20, 21, 22, 23, 1497, 1498, 1499, 1500]
    D[8:14] = [0, 19, 1501, 1600, 1, 18]
    sa = rng.integers(0, n_sa + 2, n)
    p = gen.make_sas(n_sa, cfg_id=51)
    b = gen.make_batch(n, 64, n_sa, cfg_id=51, in_len_override=D, sa_idx_override=sa)
    assert_same(gpu_run(p, [b], pipeline=pipe), oracle_run(p, [b]))


@pytest.mark.parametrize("pipe", PIPES)
def test_unaligned_packed_layout(pipe):
    """Datagrams back to back at arbitrary byte offsets (any alignment)."""
    p = gen.make_sas(9, cfg_id=52)
    bs = [gen.make_batch(3000, "imix", 9, cfg_id=52, batch=k, layout="packed") for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("pipe", PIPES)
def test_sequence_overflow(pipe):
    """RFC 4303 §3.3.3: SAs near 2^32-1 stop numbering and drop the rest."""
    n_sa = 4
    p = gen.make_sas(n_sa, cfg_id=53)
    p.seq[:] = [0xFFFFFFF0, 0xFFFFFFFF, 5, 0xFFFFFF00]
    bs = [gen.make_batch(3000, 64, n_sa, cfg_id=53, batch=k) for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("pipe", PIPES)
def test_non_default_stream(pipe):
    import torch
    s = torch.cuda.Stream()
    p = gen.make_sas(16, cfg_id=54)
    bs = [gen.make_batch(2048, "imix", 16, cfg_id=54, batch=k) for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=pipe, stream=s), oracle_run(p, bs))


def test_empty_batch_is_noop():
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    p = gen.make_sas(2, cfg_id=55)
    t = nba_ipsec.SATable(p, max_batch=16)
    z = torch.zeros(16, dtype=torch.int32, device="cuda")
    t.process(z, z, z, z, z, z, z, n=0)
    assert t.counters()["batches"] == 0
    with pytest.raises(nba_ipsec.NbaIpsecError):
        t.process(z, z, z, z, z, z, z, n=17)      # > max_batch
    t.close()


def test_virtual_shards_union_equals_oracle():
    """T7: SA-hash sharding (s mod G) across G independent tables reproduces the
    single oracle run over the same traffic (GPUs never exchange packets)."""
    from paper_conf_eurosys_kimjlmsm15_b200 import shard
    n_sa, n = 64, 8000
    p = gen.make_sas(n_sa, cfg_id=56)
    b = gen.make_batch(n, "imix", n_sa, cfg_id=56)
    (o_out, o_len), = oracle_run(p, [b])[0]
    for G in (2, 4):
        seen = np.zeros(n, bool)
        for r in range(G):
            sp, sb, idx = shard.shard_batch(p, b, r, G)
            (g_out, g_len), = gpu_run(sp, [sb])[0]
            for j, i in enumerate(idx):
                L = int(g_len[j])
                assert L == int(o_len[i])
                assert g_out[sb.out_off[j]:sb.out_off[j] + L].tobytes() == \
                    o_out[b.out_off[i]:b.out_off[i] + L].tobytes()
                seen[i] = True
        assert seen[b.sa_idx < n_sa].all()


@pytest.mark.parametrize("pipe", PIPES)
def test_last_cta_scan_fallback(pipe, monkeypatch):
    """The per-SA column scans on the last CTA (the path taken when the prologue
    grid cannot be co-resident), forced with NBA_IPSEC_NO_GRIDSYNC."""
    monkeypatch.setenv("NBA_IPSEC_NO_GRIDSYNC", "1")
    p = gen.make_sas(300, cfg_id=57)
    bs = [gen.make_batch(20000, "imix", 300, cfg_id=57, batch=k) for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=pipe), oracle_run(p, bs))


@pytest.mark.parametrize("cfg", [2, 4])
def test_two_kernel_fused_path(cfg, monkeypatch):
    """The prologue kernel + fused kernel path (used when a batch exceeds one
    super-round per CTA), forced with NBA_IPSEC_NO_MERGE at full size."""
    monkeypatch.setenv("NBA_IPSEC_NO_MERGE", "1")
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    bs = [gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg, batch=k) for k in range(2)]
    assert_same(gpu_run(p, bs, pipeline=0), oracle_run(p, bs))


def test_large_batch_uses_two_kernels():
    """n > 512 x SMs: several super-rounds per CTA behind the prologue kernel."""
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec
    n, n_sa = 100000, 700
    p = gen.make_sas(n_sa, cfg_id=58)
    bs = [gen.make_batch(n, "imix", n_sa, cfg_id=58, batch=k) for k in range(2)]
    t = nba_ipsec.SATable(p, max_batch=n)
    g = gpu_run(p, bs, table=t)
    assert t.launches_per_batch() == 2
    t.close()
    assert_same(g, oracle_run(p, bs))


def test_concurrent_tables_on_two_streams():
    """Two tables on two streams with interleaved launches (the merged kernel's
    grid barriers rely on cooperative launch for co-residency)."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    ps = [gen.make_sas(64, cfg_id=59 + k) for k in range(2)]
    bs = [[gen.make_batch(30000, "imix", 64, cfg_id=59 + k, batch=j) for j in range(3)]
          for k in range(2)]
    ts = [nba_ipsec.SATable(ps[k], max_batch=30000) for k in range(2)]
    ss = [torch.cuda.Stream() for _ in range(2)]
    dbs = [[device.to_device(b, "cuda") for b in bs[k]] for k in range(2)]
    torch.cuda.synchronize()
    for j in range(3):
        for k in range(2):
            with torch.cuda.stream(ss[k]):
                ts[k].process(*dbs[k][j].args(), n=bs[k][j].n, stream=ss[k])
    torch.cuda.synchronize()
    for k in range(2):
        res = [device.fetch(d) for d in dbs[k]]
        assert ts[k].launches_per_batch() == 1
        assert_same((res, ts[k].sa_seq(), ts[k].counters()), oracle_run(ps[k], bs[k]))
        ts[k].close()


@pytest.mark.parametrize("meta", ["in_place", "staged", "pageable"])
def test_host_buffer_path_pipelined_and_mixed(meta, monkeypatch):
    """nba_ipsec_process_batch_host (the e2e API): pinned host buffers, three
    batches in flight through the copy-in / kernels / copy-out pipeline, then a
    device-path batch and another host batch on the same table: outputs, lengths,
    counters and SA counters equal the oracle's sequential run.  The per-packet
    arrays (pinned) read / written by the kernels in place (default), staged
    by copies (forced), or staged because they are pageable."""
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    if meta == "staged":
        monkeypatch.setenv("NBA_IPSEC_HOST_META", "stage")
    pin_meta = (lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()) if meta != "pageable" \
        else (lambda a: torch.from_numpy(np.ascontiguousarray(a).copy()))
    n_sa = 48
    p = gen.make_sas(n_sa, cfg_id=60)
    bs = [gen.make_batch(5000, "imix", n_sa, cfg_id=60, batch=k, layout="packed") for k in range(5)]
    t = nba_ipsec.SATable(p, max_batch=5000)
    in_bytes = max(int(b.in_off[-1]) + int(b.in_len[-1]) for b in bs)
    out_bytes = max(int(b.out_pool_bytes) for b in bs)
    t.reserve_host_io(in_bytes, out_bytes)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
    st = torch.cuda.current_stream()
    res = [None] * 5
    hosts = []
    for k in (0, 1, 2):
        b = bs[k]
        h = dict(i=pin(b.in_buf), o=pin_meta(b.in_off.view(np.int32)), l=pin_meta(b.in_len.view(np.int16)),
                 s=pin_meta(b.sa_idx.view(np.int32)), oo=pin_meta(b.out_off.view(np.int32)),
                 out=torch.zeros(b.out_pool_bytes, dtype=torch.uint8).pin_memory(),
                 ol=pin_meta(np.zeros(b.n, dtype=np.int16)))
        hosts.append(h)
        t.process_host(h["i"], h["o"], h["l"], h["s"], h["out"], h["oo"], h["ol"],
                       int(b.in_off[-1]) + int(b.in_len[-1]), b.out_pool_bytes, n=b.n, stream=st)
    db = device.to_device(bs[3], "cuda")
    t.process(*db.args(), n=bs[3].n, stream=st)
    b = bs[4]
    h = dict(i=pin(b.in_buf), o=pin_meta(b.in_off.view(np.int32)), l=pin_meta(b.in_len.view(np.int16)),
             s=pin_meta(b.sa_idx.view(np.int32)), oo=pin_meta(b.out_off.view(np.int32)),
             out=torch.zeros(b.out_pool_bytes, dtype=torch.uint8).pin_memory(),
             ol=pin_meta(np.zeros(b.n, dtype=np.int16)))
    hosts.append(h)
    t.process_host(h["i"], h["o"], h["l"], h["s"], h["out"], h["oo"], h["ol"],
                   int(b.in_off[-1]) + int(b.in_len[-1]), b.out_pool_bytes, n=b.n, stream=st)
    t.host_wait(st)
    torch.cuda.synchronize()
    for j, k in enumerate((0, 1, 2)):
        res[k] = (hosts[j]["out"].numpy(), hosts[j]["ol"].numpy().view(np.uint16))
    res[3] = device.fetch(db)
    res[4] = (hosts[3]["out"].numpy(), hosts[3]["ol"].numpy().view(np.uint16))
    seq, ctr = t.sa_seq(), t.counters()
    t.close()
    o_res, o_seq, o_ctr = oracle_run(p, bs)
    # the host path copies the whole staging range back: only each slot's
    # [0, out_len) is defined (include/nba_ipsec.h)
    for k, b in enumerate(bs):
        (go, gl), (oo, ol) = res[k], o_res[k]
        assert np.array_equal(gl, ol), k
        for i in range(b.n):
            o, L = int(b.out_off[i]), int(ol[i])
            assert np.array_equal(go[o:o + L], oo[o:o + L]), (k, i)
    assert np.array_equal(seq, o_seq) and ctr == o_ctr
