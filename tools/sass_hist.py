#!/usr/bin/env python
"""SASS-derived per-unit work of the lane loop ("replace the
≈420 / ≈610 op estimates with cuobjdump -sass counts").

    python tools/sass_hist.py [--kernel k_fused_ring_pipe] [--out profiles/r02_sass_hist.txt]

Extracts the cubin of k_fused.cu from libnba_ipsec.so (cuobjdump -xelf), disassembles
it with line and inlining information (nvdisasm -gi; the library is built with
-lineinfo) and attributes every SASS instruction of the kernel to the source
function it was inlined from.  Per unit of algorithmic work:

  * AES-128-CTR, one 64-byte step = 4 counter blocks (aes4_keystream,
    fused_common.cuh): the instructions outside the `#pragma unroll 1` round
    loop once, the loop body x 7 (rounds 3..9);
  * SHA-1 compression (sha1_compress_fma, sha1.cuh, fully unrolled): once;
  * per packet: the CTR precompute (rounds 1-2, ctr_precompute) and the lane's
    key expansion (expand_key_lane) once.

Each instruction is assigned to the pipe it issues on (B300_MICROARCH.md
"Pipe rates": IADD3 / LOP3 / SHF / PRMT / ISETP / SEL / LEA / min-max on the
ALU pipe; IMAD* / FFMA on the FMA pipe; LDS / STS / SHFL / ATOMS on the
shared-memory (MIO) path; LDG / STG on the global LSU path).  VIADD is counted
on the ALU pipe (unverified; it appears only outside the inner loops here).
"""
from __future__ import annotations

import argparse
import collections
import glob
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_eurosys_kimjlmsm15_b200", "csrc")
SO = os.path.join(ROOT, "paper_conf_eurosys_kimjlmsm15_b200", "libnba_ipsec.so")

ALU = {"IADD3", "LOP3", "SHF", "PRMT", "ISETP", "SEL", "LEA", "IMNMX", "VIMNMX", "VIADD",
       "VIADDMNMX", "FLO", "BREV", "POPC", "PLOP3", "FMNMX", "IABS", "LEA.HI", "SGXT", "BMSK"}
FMA = {"IMAD", "FFMA", "FMUL", "FADD", "HFMA2", "IMUL", "I2F", "F2I"}
SMEM = {"LDS", "STS", "SHFL", "ATOMS", "MATCH", "LDSM"}
GMEM = {"LDG", "STG", "LD", "ST", "LDL", "STL", "RED", "REDG", "ATOMG", "ATOM", "CCTL"}
CTRL = {"BRA", "BSSY", "BSYNC", "EXIT", "WARPSYNC", "BAR", "NOP", "YIELD", "CALL", "RET",
        "ENDCOLLECTIVE", "VOTE", "BPT", "WARPGROUP"}


def pipe_of(op: str) -> str:
    base = op.split(".")[0]
    if base in ALU:
        return "alu"
    if base in FMA:
        return "fma"
    if base in SMEM:
        return "smem"
    if base in GMEM:
        return "gmem"
    if base in CTRL:
        return "ctrl"
    if base.startswith("U") or base in ("S2UR", "R2UR", "LDCU"):
        return "uniform"
    return "other"


def func_ranges(path: str, names):
    """Line ranges [start, end] of the named __device__ functions in a source file
    (from the line holding `name(` to its matching closing brace)."""
    lines = open(path).read().split("\n")
    out = {}
    for name in names:
        for i, l in enumerate(lines):
            if re.search(r"\b" + re.escape(name) + r"\s*\(", l) and "__device__" in " ".join(lines[max(0, i - 2):i + 1]):
                depth, started = 0, False
                for j in range(i, len(lines)):
                    depth += lines[j].count("{") - lines[j].count("}")
                    if "{" in lines[j]:
                        started = True
                    if started and depth == 0:
                        out[name] = (i + 1, j + 1)
                        break
                break
    return out


def disassemble(kernel: str) -> list:
    """[(opcode, [(file, line), ...innermost first])] for the kernel's SASS."""
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", SO], cwd=tmp, check=True, capture_output=True)
    cub = [c for c in glob.glob(os.path.join(tmp, "k_fused*.cubin"))][0]
    txt = subprocess.run(["nvdisasm", "-gi", cub], check=True, capture_output=True, text=True).stdout
    sec = None
    frames, pending = [], []
    out = []
    ins_re = re.compile(r"^\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)")
    loc_re = re.compile(r'//## File "([^"]+)", line (\d+)(.*)$')
    inl_re = re.compile(r'inlined at "([^"]+)", line (\d+)')
    for line in txt.split("\n"):
        if line.startswith(".text."):
            sec = line[len(".text."):].rstrip(":")
            continue
        if sec is None or kernel not in sec:
            continue
        m = loc_re.search(line)
        if m:
            # nvdisasm -gi prints one //## line per inlining level before an
            # instruction, innermost first: they accumulate into its chain
            pending.append((os.path.basename(m.group(1)), int(m.group(2))))
            pending += [(os.path.basename(f), int(n)) for f, n in inl_re.findall(m.group(3))]
            continue
        m = ins_re.match(line)
        if m:
            if pending:
                frames, pending = pending, []
            out.append((m.group(2), list(frames)))
    return out


def in_func(frames, fname, rng):
    return any(f == fname and rng[0] <= ln <= rng[1] for f, ln in frames)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kernel", default="k_fused_ring_pipe")
    ap.add_argument("--out", default=None)
    ap.add_argument("--instances", type=int, default=1,
                    help="inlined copies of the lane path in the kernel (k_fused_ring_roles: 2, its "
                         "fixed-slot and sorted-slot lanes); per-unit counts are divided by it")
    a = ap.parse_args()
    fc = os.path.join(CSRC, "fused_common.cuh")
    rfc = func_ranges(fc, ["aes4_keystream", "ctr_precompute", "expand_key_slots"])
    rsha = func_ranges(os.path.join(CSRC, "sha1.cuh"), ["sha1_compress_fma"])
    # the round loop of aes4_keystream: from its `for (int r = 0; r < 7` line to
    # the line before the final round's key load (`rkh[3 * F_THREADS`)
    src = open(fc).read().split("\n")
    a0, a1 = rfc["aes4_keystream"]
    loop0 = next(i + 1 for i in range(a0 - 1, a1) if "r < 7" in src[i])
    loop1 = next(i + 1 for i in range(loop0, a1) if "rkh[3 * F_THREADS" in src[i]) - 1
    ins = disassemble(a.kernel)
    regions = collections.OrderedDict(
        (k, collections.Counter()) for k in
        ("aes_step_outside_loop", "aes_round_loop_body", "sha1_compress", "ctr_precompute",
         "expand_key_lane", "kernel_total"))
    ops = collections.OrderedDict((k, collections.Counter()) for k in regions)
    for op, fr in ins:
        p = pipe_of(op)
        regions["kernel_total"][p] += 1
        ops["kernel_total"][op.split(".")[0]] += 1
        key = None
        if in_func(fr, "sha1.cuh", rsha["sha1_compress_fma"]):
            key = "sha1_compress"
        elif in_func(fr, "fused_common.cuh", rfc["aes4_keystream"]):
            inner = [ln for f, ln in fr if f == "fused_common.cuh" and a0 <= ln <= a1]
            key = "aes_round_loop_body" if inner and loop0 <= inner[-1] <= loop1 else "aes_step_outside_loop"
        elif in_func(fr, "fused_common.cuh", rfc["ctr_precompute"]):
            key = "ctr_precompute"
        elif in_func(fr, "fused_common.cuh", rfc["expand_key_slots"]):
            key = "expand_key_lane"
        if key:
            regions[key][p] += 1
            ops[key][op.split(".")[0]] += 1
    pipes = ("alu", "fma", "smem", "gmem", "ctrl", "uniform", "other")

    def dyn(*parts):
        c = collections.Counter()
        for k, mult in parts:
            for p, v in regions[k].items():
                c[p] += v * mult
        return c

    aes4 = dyn(("aes_step_outside_loop", 1), ("aes_round_loop_body", 7))
    per_block = {p: aes4[p] / 4.0 / a.instances for p in pipes}
    sha = {p: v / a.instances for p, v in dyn(("sha1_compress", 1)).items()}
    for k in ("ctr_precompute", "expand_key_lane"):
        regions[k] = collections.Counter({p: v / a.instances for p, v in regions[k].items()})
    lines = [f"# SASS histogram of {a.kernel} (libnba_ipsec.so, nvdisasm -gi), by source function and pipe",
             f"# aes4_keystream fused_common.cuh:{a0}-{a1} (round loop {loop0}-{loop1}, x7); "
             f"sha1_compress_fma sha1.cuh:{rsha['sha1_compress_fma'][0]}-{rsha['sha1_compress_fma'][1]}",
             "region".ljust(24) + "".join(p.rjust(9) for p in pipes) + "   top opcodes"]
    for k, c in regions.items():
        top = ", ".join(f"{o} {n}" for o, n in ops[k].most_common(8))
        lines.append(k.ljust(24) + "".join(str(c[p]).rjust(9) for p in pipes) + "   " + top)
    lines.append("")
    lines.append(f"per unit (dynamic: loop body x 7; / {a.instances} inlined copies of the lane path)")
    lines.append("AES-128 block (1/4 step)".ljust(24) + "".join(f"{per_block[p]:9.1f}" for p in pipes))
    lines.append("SHA-1 compression".ljust(24) + "".join(f"{sha.get(p, 0):9.1f}" for p in pipes))
    lines.append("per packet: ctr_precompute".ljust(24) + "".join(str(regions['ctr_precompute'][p]).rjust(9) for p in pipes))
    lines.append("per packet: key expansion".ljust(24) + "".join(str(regions['expand_key_lane'][p]).rjust(9) for p in pipes))
    summary = {"aes_block": {p: per_block[p] for p in pipes},
               "sha1_compression": {p: sha.get(p, 0) for p in pipes},
               "ctr_precompute_per_packet": dict(regions["ctr_precompute"]),
               "expand_key_per_packet": dict(regions["expand_key_lane"])}
    lines.append("")
    lines.append("JSON " + __import__("json").dumps(summary))
    text = "\n".join(lines)
    print(text)
    if a.out:
        with open(a.out, "w") as f:
            f.write(text + "\n")


if __name__ == "__main__":
    sys.exit(main())
