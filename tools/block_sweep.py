"""Loop time vs CTA size for single chains (C2's longest, C5's longest,
C3): python tools/block_sweep.py.  Needs a B200."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

for inst in (gen.config_instances("C2")[19], gen.sweep_instance(160, 4, 1), gen.sweep_instance(160, 4, 7),
             gen.config_instances("C3")[0]):
    h = dts.create(inst)
    row = []
    for b in (32, 64, 128, 256, 512):
        t = []
        for _ in range(3):
            dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, dts.dts_run_opts_default(block_threads=b))
            t.append(dts.dts_result(h).loop_ms)
        row.append(f"{b}:{min(t):.2f}")
    print(inst.name, " ".join(row), flush=True)
