"""Workloads for compute-sanitizer runs of the shipped kernels:

    compute-sanitizer --tool {memcheck,initcheck,racecheck,synccheck} \\
        python tools/sanitize_cases.py {c1,c4,ring64,roles,ring_small,inbound,inring,host}

c1         BASELINE configs[0] (64 x 64 B, 1 SA) through process_batch (k_fused<1>)
c4         configs[3] (IMIX, 65,536 packets, 1024 SAs) through process_batch
ring64     the bench's ring: 2 full-size 64-B slots (65,536 packets, 1024 SAs),
           3 batches in one run_batches (k_fused_ring_roles, then k_fused_ring_pipe)
roles      a 3,000-packet 64 B / IMIX ring in the role-split form, runs of 5 and 3
ring_small a 3,000-packet 64 B / IMIX ring in both persistent forms
inbound    ESP inbound of an IMIX batch (k_in_fused<1>) with replays and a forgery
inring     the software-pipelined inbound ring (k_in_fused_ring_pipe), 3 slots, runs of 3 and 6
host       the host-buffer path (process_batch_host), metadata read / out_len written in place
Each case checks its result against the oracle and prints one line."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec, shard  # noqa: E402


def outbound(p, batches, ring=False, slots=None, runs=(1,), form=None):
    n_sa = len(p.spi)
    sas = oracle.make_sas(p)
    n = max(b.n for b in batches)
    with nba_ipsec.SATable(p, device=0, max_batch=n) as t:
        ds = [device.to_device(b, "cuda") for b in batches]
        last = {}
        if ring:
            r = t.ring([(*d.args(), d.n) for d in ds])
            if form is not None:
                r.set_form(form)
            k = 0
            for nb in runs:
                r.run_batches(nb)
                for _ in range(nb):
                    last[k % len(ds)] = oracle.process_batch(sas, n_sa, batches[k % len(ds)])[:2]
                    k += 1
            torch.cuda.synchronize()
            r.close()
        else:
            for i, (d, b) in enumerate(zip(ds, batches)):
                t.process(*d.args(), n=b.n)
                last[i] = oracle.process_batch(sas, n_sa, b)[:2]
        ok = True
        for i, (o_out, o_len) in last.items():
            g_out, g_len = device.fetch(ds[i])
            ok &= bool(np.array_equal(g_len, o_len) and np.array_equal(g_out, o_out))
        ok &= bool(np.array_equal(t.sa_seq(), oracle.sa_seq(sas, n_sa)))
        return ok


def main():
    case = sys.argv[1]
    if case == "c1":
        c = gen.CONFIGS[1]
        p = gen.make_sas(c["n_sa"], cfg_id=1)
        ok = outbound(p, [gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=1)])
    elif case == "c4":
        p, b = shard.rank_workload(4, 65536, "imix", 1024, 0, 1)
        ok = outbound(p, [b])
    elif case == "ring64":
        p, b = shard.rank_workload(2, 65536, 64, 1024, 0, 1)
        bs = [b, gen.make_batch(65536, 64, 1024, cfg_id=2, batch=1)]
        ok = outbound(p, bs, ring=True, runs=(3,))                               # role-split (default)
        ok &= outbound(p, bs, ring=True, runs=(3,), form=nba_ipsec.Ring.PIPELINED)
    elif case == "roles":           # role-split ring, mixed lengths, runs past the record ring
        p = gen.make_sas(16, cfg_id=9)
        bs = [gen.make_batch(3000, sz, 16, cfg_id=9, batch=k) for k, sz in enumerate((64, "imix"))]
        bs[1].sa_idx[::53] = 99
        ok = outbound(p, bs, ring=True, runs=(5, 3), form=nba_ipsec.Ring.ROLES)
    elif case == "ring_small":
        p = gen.make_sas(16, cfg_id=7)
        bs = [gen.make_batch(3000, sz, 16, cfg_id=7, batch=k) for k, sz in enumerate((64, "imix"))]
        ok = outbound(p, bs, ring=True, runs=(3, 2))
        ok &= outbound(p, bs, ring=True, runs=(2, 3), form=nba_ipsec.Ring.PERSISTENT)
    elif case == "inbound":
        n, n_sa = 4000, 33
        p = gen.make_sas(n_sa, cfg_id=8)
        b = gen.make_batch(n, "imix", n_sa, cfg_id=8)
        e_out, e_len, _ = oracle.process_batch(oracle.make_sas(p), n_sa, b)
        order = np.concatenate([np.arange(n), [5, 17, 300]])
        ib = gen.esp_batch(e_out, b.out_off, e_len, b.sa_idx, order)
        ib.in_buf[ib.in_off[9] + 40] ^= 1
        sas = oracle.make_sas(p)
        win = oracle.make_windows(sas, n_sa)
        o_out, o_len, o_st, _ = oracle.process_inbound(sas, win, n_sa, ib)
        with nba_ipsec.SATable(p, device=0, max_batch=ib.n) as t:
            t.enable_inbound()
            db = device.to_device(ib, "cuda")
            st = torch.zeros(ib.n, dtype=torch.uint8, device="cuda")
            t.process_inbound(*db.args(), status=st, n=ib.n)
            g_out, g_len = device.fetch(db)
            ok = bool(np.array_equal(st.cpu().numpy(), o_st) and np.array_equal(g_len, o_len))
    elif case == "inring":          # the software-pipelined inbound ring, 3 slots x 2 runs
        os.environ["NBA_IPSEC_RING_IN_PIPE"] = "1"
        n_sa = 33
        p = gen.make_sas(n_sa, cfg_id=8)
        sas0 = oracle.make_sas(p)
        bs = []
        for k in range(3):
            b = gen.make_batch(3000, "imix", n_sa, cfg_id=8, batch=k)
            e_out, e_len, _ = oracle.process_batch(sas0, n_sa, b)
            bs.append(gen.esp_batch(e_out, b.out_off, e_len, b.sa_idx, np.arange(b.n)))
        sas = oracle.make_sas(p)
        win = oracle.make_windows(sas, n_sa)
        with nba_ipsec.SATable(p, device=0, max_batch=3000) as t:
            t.enable_inbound()
            ds = [device.to_device(ib, "cuda") for ib in bs]
            sts = [torch.zeros(ib.n, dtype=torch.uint8, device="cuda") for ib in bs]
            ring = t.ring_inbound([(*d.args(), st, ib.n) for d, st, ib in zip(ds, sts, bs)])
            ok = ring.form == ring.PIPELINED
            ring.run_batches(3)
            torch.cuda.synchronize()
            for k in range(3):                                       # first pass: all accepted
                ok &= bool(np.all(sts[k].cpu().numpy() == 0))
            ring.run_batches(6)                                      # every hash of the rotation reused
            torch.cuda.synchronize()
            for k in range(3):
                ok &= bool(np.all(sts[k].cpu().numpy() == 3))     # replayed slots: DROP_REPLAY
            ring.close()
    elif case == "host":            # the host-buffer path, metadata read / written in place
        n_sa = 48
        p = gen.make_sas(n_sa, cfg_id=60)
        bs = [gen.make_batch(5000, "imix", n_sa, cfg_id=60, batch=k, layout="packed") for k in range(3)]
        sas = oracle.make_sas(p)
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()  # noqa: E731
        with nba_ipsec.SATable(p, device=0, max_batch=5000) as t:
            t.reserve_host_io(max(int(b.in_off[-1]) + int(b.in_len[-1]) for b in bs),
                              max(int(b.out_pool_bytes) for b in bs))
            hs = []
            for b in bs:
                h = dict(i=pin(b.in_buf), o=pin(b.in_off.view(np.int32)), l=pin(b.in_len.view(np.int16)),
                         s=pin(b.sa_idx.view(np.int32)), oo=pin(b.out_off.view(np.int32)),
                         out=torch.zeros(b.out_pool_bytes, dtype=torch.uint8).pin_memory(),
                         ol=torch.zeros(b.n, dtype=torch.int16).pin_memory())
                t.process_host(h["i"], h["o"], h["l"], h["s"], h["out"], h["oo"], h["ol"],
                               int(b.in_off[-1]) + int(b.in_len[-1]), b.out_pool_bytes, n=b.n)
                hs.append(h)
            t.host_wait()
            torch.cuda.synchronize()
            ok = True
            for h, b in zip(hs, bs):
                o_out, o_len, _ = oracle.process_batch(sas, n_sa, b)
                gl = h["ol"].numpy().view(np.uint16)
                ok &= bool(np.array_equal(gl, o_len))
                go = h["out"].numpy()
                for i in range(b.n):
                    o, L = int(b.out_off[i]), int(o_len[i])
                    ok &= bool(np.array_equal(go[o:o + L], o_out[o:o + L]))
    else:
        raise SystemExit(f"unknown case {case}")
    print(f"{case}: result == oracle: {ok}", flush=True)


if __name__ == "__main__":
    main()
