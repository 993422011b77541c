"""Repeat the full C5 batched sweep (optionally under compute-sanitizer) and
check every repetition gives the same schedules.  Needs a B200.
usage: python tools/san_c5.py [reps] [every]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 4
every = int(sys.argv[2]) if len(sys.argv) > 2 else 1
insts = gen.config_instances("C5")[::every]
hs = [dts.create(i) for i in insts]
o = dts.dts_run_opts_default(flags=dts.DTS_F_FALLBACK2)
ref = None
for r in range(reps):
    dts.dts_sweep_run(hs, dts.DTS_POLICY_DARTS_LUF, o)
    res = [dts.dts_result(h) for h in hs]
    sig = [(g.n_served, g.n_loads, g.makespan) for g in res]
    if ref is None:
        ref = sig
    assert sig == ref, f"rep {r}: results differ"
    assert all(g.n_served == i.m for g, i in zip(res, insts))
    print("rep", r, "ok", flush=True)
print("C5 repeated sweeps ok:", len(insts), "instances x", reps)
