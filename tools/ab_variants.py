"""A/B compile-time variants of libnba_ipsec.so on the same GPU box.

    python tools/ab_variants.py build NAME=DEF1,DEF2 NAME2=...   (here: nvcc only)
    python tools/ab_variants.py run [cfg ...]                    (GPU: time every variant)

Variants are written to build/variants/<name>.so; `run` times each one in a
fresh process (bench protocol: L2 flush, per-step events) through the
NBA_IPSEC_LIB override, interleaving variants twice to expose drift."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VDIR = os.path.join(ROOT, "build", "variants")
sys.path.insert(0, ROOT)

TIMER = r'''
import os, sys
sys.path.insert(0, %r)
sys.path.insert(0, %r)
import torch
from paper_conf_eurosys_kimjlmsm15_b200 import device, gen, nba_ipsec
from ab_merge import timed
for cfg in %r:
    c = gen.CONFIGS[cfg]
    p = gen.make_sas(c["n_sa"], cfg_id=cfg)
    b = gen.make_batch(c["n"], c["size"], c["n_sa"], cfg_id=cfg)
    db = device.to_device(b, "cuda")
    t = nba_ipsec.SATable(p, max_batch=c["n"])
    print(f"  cfg {cfg}: {timed(t, db, b.n):.1f} us/step", flush=True)
    t.close()
'''


def main():
    if sys.argv[1] == "build":
        from paper_conf_eurosys_kimjlmsm15_b200 import build
        os.makedirs(VDIR, exist_ok=True)
        for spec in sys.argv[2:]:
            name, _, defs = spec.partition("=")
            d = [x for x in defs.split(",") if x]
            print(name, build.build(out=os.path.join(VDIR, name + ".so"), defines=d))
        return
    cfgs = [int(x) for x in sys.argv[2:]] or [2, 3, 4]
    names = sorted(f[:-3] for f in os.listdir(VDIR) if f.endswith(".so"))
    code = TIMER % (ROOT, os.path.join(ROOT, "tools"), cfgs)
    for rep in range(2):
        for n in names:
            print(f"variant {n} (pass {rep})", flush=True)
            env = dict(os.environ, NBA_IPSEC_LIB=os.path.join(VDIR, n + ".so"))
            subprocess.run([sys.executable, "-c", code], env=env, check=True)


if __name__ == "__main__":
    main()
