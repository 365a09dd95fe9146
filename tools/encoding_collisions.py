"""Exp #5 analog (Fig 13) without the model: how many feature IDs share a
flat key under short flat keys, size-aware (reading R24) vs fixed-length ("Kraken",
P:L632-639), for the Criteo Kaggle (cfg2) and Terabyte (cfg3) table sizes.  Uses the
oracle's encoders (test infrastructure).  For a hashed table with c rows in 2^g codes the
expected fraction of rows that share their code is 1 - (1 - 2^-g)^(c-1); exact tables
contribute 0.  Reported: row-weighted colliding fraction and the number of lossy tables.

python tools/encoding_collisions.py > profiles/encoding_collisions_r01.json
"""
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from oracle import oracle as O  # noqa: E402
from workload import configs  # noqa: E402


def colliding(cards, bits, ex):
    rows = sum(cards)
    col = 0.0
    for c, g, e in zip(cards, bits, ex):
        if not e and c > 1:
            col += c * (1.0 if g == 0 else 1.0 - math.exp((c - 1) * math.log1p(-2.0 ** -int(g))))
    return col / rows


out = {"what": __doc__.split("\n")[0], "configs": {}}
for name in ("cfg2", "cfg3"):
    w = configs.get(name)
    bmin = O.encode(w.cards)[0]
    rows = []
    for B in range(16, 33):
        r = {"key_bits": B}
        for kind, fixed in (("size_aware", False), ("fixed_length", True)):
            lossy, base, bits, ex = O.encode_short(w.cards, B, fixed=fixed)
            r[kind] = None if lossy < 0 else {"lossy_tables": int(lossy),
                                               "colliding_row_fraction": colliding(w.cards, bits, ex)}
        rows.append(r)
    out["configs"][name] = {"tables": w.n, "rows": int(sum(w.cards)), "bmin_exact": bmin, "by_key_bits": rows}
print(json.dumps(out, indent=1))
