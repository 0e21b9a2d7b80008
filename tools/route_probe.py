"""route_pack / route_dispatch on the bench's 64-B batch (8 owners), for ncu launch lists."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec, redistribute  # noqa: E402

b = gen.make_batch(65536, 64, 1024, cfg_id=2)
db = device.to_device(b, "cuda")
cap_b = int(b.in_len.astype(np.int64).sum()) + 64
rxs = [redistribute.alloc_rx(b.n, cap_b, "cuda") for _ in range(8)]
table = redistribute.rx_table(rxs, "cuda")
ws = torch.empty(nba_ipsec.route_workspace_bytes(b.n, 8), dtype=torch.uint8, device="cuda")
dc = torch.zeros(9, dtype=torch.int64, device="cuda")
dbyt = torch.zeros(9, dtype=torch.int64, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for k in range(6):
    e0.record()
    nba_ipsec.route_dispatch(db.in_buf, db.in_off, db.in_len, db.sa_idx, b.n, 1024, None, 8, ws,
                             table, b.n, cap_b, dc, dbyt)
    e1.record()
    torch.cuda.synchronize()
    print(f"dispatch {e0.elapsed_time(e1) * 1e3:.1f} us")
