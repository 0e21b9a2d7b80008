"""Host plumbing (no GPU): the device tree of the adaptive split, the receive
descriptor table of the peer-memory dispatch, and the one-process views of
packed owner regions -- checked on CPU tensors against their plain statements."""
import numpy as np
import torch

from oracle import alb as oalb
from paper_conf_eurosys_kimjlmsm15_b200 import alb, nba_ipsec, redistribute


def test_internal_nodes_cover_every_device_once():
    for n_dev in range(1, 9):
        nodes = alb.internal_nodes(n_dev)
        assert len(nodes) == n_dev - 1                   # a binary tree over n leaves
        assert all(nid < nba_ipsec.ALB_TREE_NODES for nid, _, _ in nodes)
        # every device is reachable: the oracle's assignment with all-middle
        # steps gives every device some SAs
        owner = oalb.assign(64 * n_dev, n_dev, [2] * 15, 4)
        assert sorted(set(owner)) == list(range(n_dev))


def test_balancer_eight_devices_moves_load_off_a_slow_device():
    """Device 7 four times slower: after enough observations the root and the
    node above device 7 have moved SAs away from it (fewer than its even share)."""
    n_sa = 1024
    b = alb.Balancer(n_sa, 8, steps=25, init_step=12, history=8, update_ns=100, wait_min=1,
                     wait_max=2)
    t = 0
    for _ in range(4000):
        owner, _ = b.assignment()
        share = np.bincount(owner, minlength=8).astype(np.int64)
        dt = [int(10 * max(share[d], 1) * (4 if d == 7 else 1)) for d in range(8)]
        t += max(dt)
        b.observe(t, dt, share.tolist())
    owner, _ = b.assignment()
    share = np.bincount(owner, minlength=8)
    assert share[7] < n_sa // 8
    assert share.sum() == n_sa


def test_rx_table_layout_and_local_views_on_cpu():
    rxs = [redistribute.alloc_rx(8, 256, "cpu") for _ in range(3)]
    tab = redistribute.rx_table(rxs, "cpu").view(3, 5)
    for r, row in zip(rxs, tab.tolist()):
        assert row == [r.buf.data_ptr(), r.off.data_ptr(), r.length.data_ptr(), r.sa.data_ptr(),
                       r.count.data_ptr()]
    # packed owner regions: 2 + 0 + 3 packets
    lens = np.array([5, 7, 1, 2, 3], np.int16)
    p = redistribute.Packed(buf=torch.arange(64, dtype=torch.uint8), length=torch.from_numpy(lens),
                            sa=torch.arange(5, dtype=torch.int32), counts=[2, 0, 3],
                            nbytes=[12, 0, 6])
    n, in_off, ln, sa, out_off, out_len, out_buf = redistribute.local_views(p, 2)
    assert n == 3
    assert in_off[:3].tolist() == [12, 13, 15]            # after owner 0's 12 bytes
    assert ln[:3].tolist() == [1, 2, 3] and sa[:3].tolist() == [2, 3, 4]
    assert out_off[:3].tolist() == [0, 65, 131]           # len + 64 per output slot
    n0, in_off0, *_ = redistribute.local_views(p, 0)
    assert n0 == 2 and in_off0[:2].tolist() == [0, 5]
    assert redistribute.local_views(p, 1)[0] == 0
