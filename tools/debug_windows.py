"""Find the first random trace / litmus whose windowed GPU race list differs from the oracle; dump it."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import oracle, paper_conf_pldi_eizenbergppmd17_b200 as bc
from bcgen.fuzz import random_trace
import litmus

def tup(r):
    return (int(r["addr"]), int(r["prior_event"]), int(r["cur_event"]), int(r["kind"]), int(r["cls"]), int(r["space"]), int(r["block"]))

out = []
cases = [(f"lit_{n}", b) for n, b, _, _ in litmus.SUITE]
cases += [(f"rnd_{s}", s) for s in range(5000, 5040)]
for we in (16, 64):
    for name, b in cases:
        if name.startswith("lit"):
            tb = b(); recs, geom = tb.records(), tb.geom.as_dict()
        else:
            recs, tb = random_trace(b); geom = tb.geom.as_dict()
        st, want, _ = oracle.detect_geom(recs, geom)
        res = bc.detect(recs, geom, device="cuda:0", window_events=we)
        if st != res.status or len(want) != len(res.races) or not np.array_equal(want.view(np.uint8), res.races.view(np.uint8)):
            W = set(map(tup, want)); G = set(map(tup, res.races))
            out.append(dict(name=name, we=we, n=len(recs), st=[st, res.status], n_want=len(want), n_got=len(res.races),
                            extra=sorted(G - W)[:40], missing=sorted(W - G)[:40], stats={k: v for k, v in res.stats.items() if k != "ms_kernel"}))
            np.save(f"gpurun_out/dbg_{name}_{we}.npy", recs)
            json.dump(geom, open(f"gpurun_out/dbg_{name}_{we}.json", "w"))
            print(name, we, "MISMATCH", len(want), len(res.races), flush=True)
json.dump(out, open("gpurun_out/dbg_windows.json", "w"), indent=1)
print(len(out), "mismatches")
