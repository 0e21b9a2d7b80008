"""Loader for tests/golden/*.txt fixtures (records of 'field = hex' lines)."""
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(fname):
    recs, cur = [], {}
    with open(os.path.join(GOLDEN, fname)) as f:
        for raw in f:
            line = raw.rstrip("\n")
            if line.startswith("#"):
                continue
            if not line.strip():
                if cur:
                    recs.append(cur)
                    cur = {}
                continue
            k, _, v = line.partition("=")
            cur[k.strip()] = v.strip()
    if cur:
        recs.append(cur)
    return {r["name"]: r for r in recs}


def msg_of(rec):
    if "msg_hex" in rec:
        m = bytes.fromhex(rec["msg_hex"])
    else:
        m = rec.get("msg_ascii", "").encode()
    return m * int(rec.get("repeat", "1"))
