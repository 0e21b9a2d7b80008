"""Per-CTA phase timeline of the fused kernel (needs NBA_IPSEC_TRACE=1)."""
import os
import sys

os.environ.setdefault("NBA_IPSEC_TRACE", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec  # noqa: E402

FLUSH = "--flush" in sys.argv
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda") if FLUSH else None
for cfg in [int(x) for x in sys.argv[1:] if x.isdigit()] or (2, 3, 4):
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg)
    t = nba_ipsec.SATable(p, max_batch=c["n"])
    db = device.to_device(b, "cuda")
    for _ in range(5):
        if flush is not None:
            flush.zero_()
        t.process(*db.args(), n=b.n)
    torch.cuda.synchronize()
    full = t.debug_trace(148).astype(np.int64)
    pro = full[-1]
    tr = full[:-1]
    live = tr[:, 0] > 0
    tr = tr[live]
    t0 = pro[0] if pro[0] > 0 else tr[:, 0].min()
    if pro[0] > 0 and pro[1] > 0:      # two-kernel path: the prologue kernel's own stamps
        print("prologue kernel: first start 0, tiles done %.2f, last-CTA start %.2f, end %.2f us" %
              ((pro[1] - t0) / 1e3, (pro[2] - t0) / 1e3, (pro[3] - t0) / 1e3))
    else:                              # one-kernel path: the prologue runs inside k_fused
        print("prologue: inside the fused kernel (one launch); phases below")
    rel = (tr - t0) / 1000.0
    names = ["start", "meta_done/arrived(merged)", "tables_done", "lanes_done", "m_tiles_done", "m_bar1_done",
             "m_scans_done", "keys_staged(tid0) / polls done (merged)"]
    print(f"config {cfg} ({c['name']}), {live.sum()} CTAs, times in us from the prologue's first "
          f"CTA start{' (L2 flushed before the batch)' if FLUSH else ''}")
    for k, nm in enumerate(names):
        col = rel[:, k]
        print(f"  {nm:12s} min {col.min():8.2f}  med {np.median(col):8.2f}  max {col.max():8.2f}")
    ld = rel[:, 3]
    print("  lanes_done percentiles:", np.percentile(ld, [10, 25, 50, 75, 90, 95, 99]).round(1))
    idx = np.nonzero(live)[0]
    order = np.argsort(-ld)[:8]
    print("  slowest CTAs (index: lanes_done / meta_done us):",
          ", ".join(f"{idx[k]}: {ld[k]:.1f}/{rel[k, 1]:.1f}/polls {rel[k, 7]:.1f}" for k in order))
    from paper_conf_eurosys_kimjlmsm15_b200 import nba_ipsec as nbm
    import ctypes
    raw = np.zeros(148 * 8 + 64, np.uint64)
    nbm.lib.nba_ipsec_debug_trace(t._h, raw.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), raw.size)
    for k, nm in ((0, "tid0 (shortest)"), (8, "last (longest)")):
        v = [int(x) for x in raw[148*8+8+k:148*8+8+k+5]]
        print("  lane %s cycles: setup %d  aes0 %d  emit0 %d  sha0 %d  rest %d" % (nm, *v))
    raw2 = np.zeros(148 * 8 + 64, np.uint64)
    nbm.lib.nba_ipsec_debug_trace(t._h, raw2.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), raw2.size)
    G = int(live.sum()) if pro[0] == 0 else 148
    kend = int(raw2[148 * 8 + 48])
    if kend:
        print("  kernel: last CTA end %.2f us after the first CTA start" % ((kend - t0) / 1e3))
    wend = raw2[148 * 8 + 24:148 * 8 + 40].astype(np.int64)
    st0 = int(full[0, 0])
    print("  CTA 0 warp finish (us from its start):", " ".join(f"{(x - st0) / 1e3:.1f}" if x else "-" for x in wend))
    t.close()
