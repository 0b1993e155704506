"""Sweep the packed inspector's routing knobs on one config: FASTZ_PAIR_LONG (predicted bases from which a side runs
in the 32-bit inspector) and FASTZ_PAIR_ESCAPE (strips after which a packed side is redone in 32 bits).
usage: python tools/pair_sweep.py <config_id> [long,...] [escape,...]   (GPU; prints one JSON line per setting)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_gundaboluvt21_b200 import fastz  # noqa: E402
from synth import genome  # noqa: E402

cid = int(sys.argv[1])
longs = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [96]
escs = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [16]
w = genome.make(cid)
for esc in escs:
    os.environ["FASTZ_PAIR_ESCAPE"] = str(esc)
    with fastz.Aligner(w.T, w.Q) as al:
        for lg in longs:
            os.environ["FASTZ_PAIR_LONG"] = str(lg)
            ms = []
            for _ in range(3):
                al.extend_only(w.seeds)
                st = al.stats()
                ms.append(st["ms_inspect"])
            print(json.dumps({"config": cid, "escape": esc, "long": lg, "ms_inspect": min(ms[1:]),
                              "packed": st["n_packed_sides"], "long_sides": st["n_long_sides"],
                              "redo": st["n_redo_sides"]}), flush=True)
