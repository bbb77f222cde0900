"""Write full-size oracle race lists under tests/golden/ (test infrastructure).

    python tools/make_golden.py c4            # BASELINE configs[3] at full size (seed 4)
    python tools/make_golden.py c2_inj c3_inj # injected variants

Calls only oracle/ (the CPU oracle, plain C++ on uncompressed vector clocks) on traces from
bcgen (the seeded input generators, which hold none of the method's arithmetic).  No value here
comes from the CUDA path.  Each output file holds the oracle's canonical race list as text, one
race per line (addr prior_event cur_event kind cls space block, hex / decimal), plus a header
with the trace's record / event counts and the oracle's wall time, so a test can check it is
comparing against the same trace.
"""
from __future__ import annotations

import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bcgen  # noqa: E402
import oracle  # noqa: E402
from bcgen.configs import ConfigPlan  # noqa: E402

# name -> (config index, generator overrides); the overrides are the ones the GPU tests use
GOLDEN = {
    "c4": (4, {}),
    "c2_inj": (2, dict(inject=1)),
    "c3_inj": (3, dict(inject=1, n_blocks=256)),
}


def write(name):
    cfg, kw = GOLDEN[name]
    plan = ConfigPlan(cfg, **kw)
    recs = plan.records()
    geom = plan.geometry
    plan.close()
    le, ce = bcgen.count_events(recs)
    t0 = time.time()
    st, races, _ = oracle.detect_geom(recs, geom)
    dt = time.time() - t0
    assert st == 0, st
    path = os.path.join(ROOT, "tests", "golden", f"{name}_oracle_races.txt")
    with open(path, "w") as f:
        f.write(f"# oracle race list, written by tools/make_golden.py {name} (oracle/ only)\n")
        f.write(f"# config={cfg} overrides={kw} records={len(recs)} lane_events={le} control_events={ce} "
                f"races={len(races)} oracle_seconds={dt:.1f}\n")
        for r in races:
            f.write(f"{int(r['addr']):x} {int(r['prior_event']):x} {int(r['cur_event']):x} "
                    f"{int(r['kind'])} {int(r['cls'])} {int(r['space'])} {int(r['block'])}\n")
    print(name, len(recs), "records", le + ce, "events", len(races), "races", f"{dt:.1f}s", flush=True)


if __name__ == "__main__":
    for n in sys.argv[1:]:
        write(n)
