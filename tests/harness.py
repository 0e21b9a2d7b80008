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
