"""Probe gstm_ubench_mix programs phase by phase: which
part of a transaction's op mix sets the roof.  GPU only.

    python tools/roof_probe.py [--layout paired|split] [--words 1048576] [--bits 20]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_xuwglgq14_b200 import build as B  # noqa: E402

B.build()
from paper_conf_cgo_xuwglgq14_b200 import gstm as G  # noqa: E402
from paper_conf_cgo_xuwglgq14_b200 import roofline as R  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--layout", default="paired")
    ap.add_argument("--words", type=int, default=1 << 20)
    ap.add_argument("--bits", type=int, default=20)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    paired = a.layout == "paired"
    h = G.Gstm(a.words, a.bits, paired=paired)
    ph = R.ph
    progs = {
        "ld2": [ph(R.LD_V, 2)],
        "ld2_ld2": [ph(R.LD_V, 2), ph(R.LD_V, 2, 2)],
        "ld2_atom2": [ph(R.LD_V, 2), ph(R.ATOM_L, 2)],
        "ld2_atom2_clock": [ph(R.LD_V, 2), ph(R.ATOM_L, 2), ph(R.CLOCK)],
        "ld2_atom2_st2": [ph(R.LD_V, 2), ph(R.ATOM_L, 2), ph(R.ST_L, 2)],
        "bank_full": [ph(R.LD_V, 2), ph(R.ATOM_L, 2), ph(R.CLOCK), ph(R.ST_L, 2)],
        "clock_only": [ph(R.CLOCK)],
        "atom2_clock_st2": [ph(R.ATOM_L, 2), ph(R.CLOCK), ph(R.ST_L, 2)],
        "atom2_clock": [ph(R.ATOM_L, 2), ph(R.CLOCK)],
        "atom2": [ph(R.ATOM_L, 2)],
    }
    full = progs["bank_full"]
    mixes = {k: R.mix([(1, q)]) for k, q in progs.items()}
    mixes["mix96_ro4"] = R.mix([(0.96, full), (0.04, [ph(R.LD_V, 2)])])
    mixes["mix_same_same"] = R.mix([(0.5, full), (0.5, full)])
    mixes["mix_4x_same"] = R.mix([(0.25, full)] * 4)
    out = []
    for name, prog in mixes.items():
        for w in (8, 16, 32, 64):
            th = 148 * 32 * w
            tps, ms = G.gstm_ubench_mix(h.h, a.words, prog, 1 << 22, th)
            r = {"prog": name, "warps_per_sm": w, "tx_per_s": tps, "ms": ms,
                 "ns_per_tx_per_thread": th / tps * 1e9}
            out.append(r)
            print(json.dumps(r), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            for r in out:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
