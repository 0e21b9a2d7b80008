"""Test harness: run the CUDA path (through the C ABI) and the oracle on the
same seeded inputs and compare.  Tests only."""
import numpy as np

import oracle
from paper_conf_eurosys_kimjlmsm15_b200 import gen


def oracle_run(params, batches, n_threads=8):
    """Sequence of batches through the oracle from params' initial state."""
    n_sa = len(params.spi)
    sas = oracle.make_sas(params)
    res = []
    ctr = oracle.Counters()
    for b in batches:
        out, ol, _ = oracle.process_batch(sas, n_sa, b, n_threads=n_threads, counters=ctr)
        res.append((out, ol.copy()))
    return res, oracle.sa_seq(sas, n_sa), ctr.as_dict()


def gpu_run(params, batches, pipeline=None, stream=None, max_batch=None, table=None):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    mb = max_batch or max(max(b.n for b in batches), 1)
    t = table or nba_ipsec.SATable(params, device=0, max_batch=mb)
    if pipeline is not None:
        t.set_pipeline(pipeline)
    res = []
    for b in batches:
        db = device.to_device(b, "cuda")
        if stream is not None:
            with torch.cuda.stream(stream):
                t.process(*db.args(), n=b.n, stream=stream)
            stream.synchronize()
        else:
            t.process(*db.args(), n=b.n)
        res.append(device.fetch(db))
    seq = t.sa_seq()
    ctr = t.counters()
    if table is None:
        t.close()
    return res, seq, ctr


def assert_same(gpu, orc):
    (g_res, g_seq, g_ctr), (o_res, o_seq, o_ctr) = gpu, orc
    for bi, ((go, gl), (oo, ol)) in enumerate(zip(g_res, o_res)):
        assert np.array_equal(gl, ol), f"batch {bi}: out_len differs at " \
            f"{np.nonzero(gl != ol)[0][:10]}"
        if not np.array_equal(go, oo):
            d = np.nonzero(go != oo)[0]
            raise AssertionError(f"batch {bi}: {d.size} output bytes differ, first at {d[:8]}")
    assert np.array_equal(g_seq, o_seq), "final SA sequence numbers differ"
    assert g_ctr == o_ctr, (g_ctr, o_ctr)


def expected_seq_numbers(params, batch):
    """Plain counting (not the oracle): seq the i-th valid packet of SA s gets."""
    n_sa = len(params.spi)
    seq = params.seq.astype(np.int64).copy()
    q = np.zeros(batch.n, np.int64)
    for i in range(batch.n):
        s = int(batch.sa_idx[i])
        D = int(batch.in_len[i])
        if s < n_sa and 20 <= D <= 1500 and seq[s] < 0xFFFFFFFF:
            seq[s] += 1
            q[i] = seq[s]
    return q, seq


# --- ESP inbound ---------------------------------------------

def esp_source(params, n, size, cfg_id, n_threads=8, batch=0):
    """Outbound ORACLE run over a gen batch: the ESP packets inbound tests feed in."""
    n_sa = len(params.spi)
    b = gen.make_batch(n, size, n_sa, cfg_id=cfg_id, batch=batch)
    sas = oracle.make_sas(params)
    out, ol, _ = oracle.process_batch(sas, n_sa, b, n_threads=n_threads)
    return b, out, ol


def oracle_inbound_run(params, batches):
    n_sa = len(params.spi)
    sas = oracle.make_sas(params)
    win = oracle.make_windows(sas, n_sa)
    ctr = oracle.InCounters()
    res = []
    for b in batches:
        out, ol, st, _ = oracle.process_inbound(sas, win, n_sa, b, counters=ctr)
        res.append((out, ol.copy(), st.copy()))
    top, bmp = oracle.window_state(win, n_sa)
    return res, (top, bmp), ctr.as_dict()


def gpu_inbound_run(params, batches, max_batch=None, out_fill=0xA5):
    import torch
    from paper_conf_eurosys_kimjlmsm15_b200 import device, nba_ipsec
    mb = max_batch or max(max(b.n for b in batches), 1)
    t = nba_ipsec.SATable(params, device=0, max_batch=mb)
    t.enable_inbound()
    res = []
    for b in batches:
        db = device.to_device(b, "cuda", out_fill=out_fill)
        st = torch.full((max(b.n, 1),), 0xEE, dtype=torch.uint8, device="cuda")
        t.process_inbound(*db.args(), status=st, n=b.n)
        out, ol = device.fetch(db)
        res.append((out, ol, st[:b.n].cpu().numpy()))
    win = t.replay_window()
    ctr = t.in_counters()
    t.close()
    return res, win, ctr


def assert_same_inbound(gpu, orc, batches):
    (g_res, g_win, g_ctr), (o_res, o_win, o_ctr) = gpu, orc
    for bi, (b, (go, gl, gs), (oo, ol, os_)) in enumerate(zip(batches, g_res, o_res)):
        if not np.array_equal(gs, os_):
            d = np.nonzero(gs != os_)[0]
            raise AssertionError(f"batch {bi}: status differs at {d[:10]}: gpu {gs[d[:10]]} "
                                 f"oracle {os_[d[:10]]}")
        assert np.array_equal(gl, ol), f"batch {bi}: out_len differs at {np.nonzero(gl != ol)[0][:10]}"
        for i in np.nonzero(ol)[0]:
            o, L = int(b.out_off[i]), int(ol[i])
            if not np.array_equal(go[o:o + L], oo[o:o + L]):
                raise AssertionError(f"batch {bi}: packet {i} inner bytes differ")
    assert np.array_equal(g_win[0], o_win[0]), "window right edges differ"
    assert np.array_equal(g_win[1], o_win[1]), "window bitmaps differ"
    assert g_ctr == o_ctr, (g_ctr, o_ctr)
