"""The bench's algorithmic work model (the roofline numerators)
against SURVEY.md Appendix B's per-size table (computed there from the RFC
formulas), and the IMIX composition of the generator (PAPER.md:603 sizes,
7:4:1 mix) -- no GPU needed."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_eurosys_kimjlmsm15_b200 import gen  # noqa: E402

# L -> (AES blocks, SHA-1 compressions inner + outer, out IP length)
APPENDIX_B = {64: (4, 3, 100), 128: (8, 4, 164), 256: (16, 6, 292), 512: (32, 10, 548),
              594: (37, 11, 632), 1024: (64, 18, 1060), 1514: (94, 25, 1552)}


def test_work_model_per_packet_matches_appendix_b():
    for L, (blocks, comps, out_len) in APPENDIX_B.items():
        b = gen.make_batch(10, L, 4, cfg_id=1)
        w = bench.work_model(b)
        assert w["packets"] == 10
        assert w["aes_blocks"] == 10 * blocks, L
        assert w["sha1_compressions"] == 10 * comps, L
        assert w["bytes_out"] == 10 * out_len, L


def test_work_model_batch_totals_match_appendix_b():
    # per 64K batch: AES threads and SHA-1 compressions
    expect = {64: (262144, 196608), 1514: (6160384, 1638400), "imix": (1474609, 491532)}
    for size, (blocks, comps) in expect.items():
        b = gen.make_batch(65536, size, 1024, cfg_id=2)
        w = bench.work_model(b)
        assert (w["aes_blocks"], w["sha1_compressions"]) == (blocks, comps), size


def test_imix_composition_and_invalid_packets_excluded():
    b = gen.make_batch(65536, "imix", 1024, cfg_id=4)
    L = np.asarray(b.frame_len)
    assert sorted(np.unique(L).tolist()) == [64, 594, 1514]
    assert [int((L == x).sum()) for x in (64, 594, 1514)] == [38229, 21845, 5462]
    b.in_len[:3] = [19, 1501, 0]                      # dropped by the path: no work
    w = bench.work_model(b)
    assert w["packets"] == 65536 - 3


def test_roofline_arithmetic():
    """ALU / LDS / HBM fractions from the SASS per-unit counts (profiles/r02d_sass_hist.txt)."""
    w = {"aes_blocks": 1000, "sha1_compressions": 100, "hbm_bytes": 5000}
    peaks = {"sm_max_mhz": 1965.0, "hbm_gbs": 6500.0, "source": "test"}
    units = bench.sass_units()
    r = bench.roofline(0.001, w, peaks, units)
    ops = 1000 * units["aes_block"]["alu"] + 100 * units["sha1_compression"]["alu"]
    assert abs(r["alu"]["achieved"] - ops / 1e-6 / 1e12) < 1e-9
    assert abs(r["alu"]["peak"] - 148 * 64 * 1965e6 / 1e12) < 1e-9
    assert abs(r["lds"]["achieved"] - 1000 * units["aes_block"]["smem"] / 1e-6 / 1e12) < 1e-9
    assert abs(r["hbm"]["achieved"] - 5000 / 1e-6 / 1e9) < 1e-9
    for k in ("alu", "lds", "hbm"):
        assert abs(r[k]["frac"] - r[k]["achieved"] / r[k]["peak"]) < 1e-12


def test_sass_units_committed():
    """The committed SASS histogram parses and gives plausible per-unit counts:
    an AES block needs its table lookups (>= 133 after the CTR precompute, at
    most 160) and a SHA-1 compression >= 80 rounds x 3 ALU ops."""
    u = bench.sass_units()
    assert u["source"].startswith("profiles/")
    assert 133 <= u["aes_block"]["smem"] <= 165
    assert u["sha1_compression"]["alu"] + u["sha1_compression"]["fma"] >= 400


def test_ring_slot_count_matches_bench_rule():
    from paper_conf_eurosys_kimjlmsm15_b200 import device
    b = gen.make_batch(65536, 64, 1024, cfg_id=2)
    R = device.ring_slot_count(b.in_len, b.n, 126 << 20)
    touched = int(b.in_len.astype(np.int64).sum()) + b.n * 323
    assert (R - 1) * touched < 2 * (126 << 20) <= R * touched


def test_bench_args_and_gpus_contract():
    a = bench.parse_args(["--gpus", "2", "--steps", "7", "--warmup", "1"])
    assert (a.gpus, a.steps, a.warmup) == (2, 7, 3)          # W >= 3


def test_gpus_n_relaunches_under_torchrun(monkeypatch):
    """`bench.py --gpus N` without a torchrun environment re-executes itself
    under torch.distributed.run with one process per GPU on 127.0.0.1 (the
    driver's form), NCCL init logging on; fewer visible GPUs fail loudly."""
    import pytest
    calls = []
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(bench.os, "execvpe", lambda f, argv, env: calls.append((argv, env)))
    import torch
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 8)
    monkeypatch.setattr(bench.sys, "argv", ["bench.py", "--gpus", "4", "--steps", "5"])
    bench.relaunch_under_torchrun(bench.parse_args(["--gpus", "4", "--steps", "5"]))
    argv, env = calls[0]
    assert argv[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=4" in argv and "127.0.0.1" in argv
    assert argv[-4:] == ["--gpus", "4", "--steps", "5"] and argv[-5].endswith("bench.py")
    assert env["NCCL_DEBUG"] == "INFO"
    monkeypatch.setattr(torch.cuda, "device_count", lambda: 1)
    with pytest.raises(SystemExit):
        bench.relaunch_under_torchrun(bench.parse_args(["--gpus", "4"]))


def test_ctx_rejects_world_mismatch(monkeypatch):
    """A rank whose WORLD_SIZE differs from --gpus refuses to run (no silent
    single-GPU number reported as N GPUs)."""
    import pytest
    monkeypatch.setenv("WORLD_SIZE", "2")
    with pytest.raises(SystemExit):
        bench.Ctx(bench.parse_args(["--gpus", "4"]))
