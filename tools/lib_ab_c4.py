"""Same-box A/B of library builds on the single large instances:
python tools/lib_ab_c4.py LIB.so [flags...]  (loop ms of C4b, C4a, C3, C2[19];
best of 2; flags are extra DTS_F_* bits, e.g. 32 = DTS_F_GENERIC)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

lib = sys.argv[1]
extra = int(sys.argv[2]) if len(sys.argv) > 2 else 0
dts.load_library(lib)
import gen  # noqa: E402

out = []
for cfg, idx, reps in (("C4b", 0, 2), ("C4a", 0, 2), ("C3", 0, 3), ("C2", 19, 7)):
    h = dts.create(gen.config_instances(cfg)[idx])
    o = dts.dts_run_opts_default(flags=dts.DTS_F_FALLBACK2 | extra)
    t = []
    for _ in range(reps):
        dts.dts_run(h, dts.DTS_POLICY_DARTS_LUF, o)
        t.append(dts.dts_result(h).loop_ms)
    out.append(f"{cfg}[{idx}] {min(t):.2f} ms")
print(f"{os.path.basename(lib)} flags+{extra}: " + "  ".join(out), flush=True)
