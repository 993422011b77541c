"""Exchange cost of the task-sharded single instance (dts_shard_group_run):
loop time, exchanges, and thread-0 cycles inside xch_sync per exchange.  Needs a B200."""
import os
os.environ.setdefault("DTS_PROFILE", "1")
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ipps_gonthiermt22_b200 as dts  # noqa: E402

cases = [gen.config_instances("C3")[0], gen.config_instances("C2")[19]]
if len(sys.argv) > 1 and sys.argv[1] == "big":
    cases = [gen.config_instances("C4b")[0]]
for inst in cases:
    for G in (1, 2, 4, 8):
        dts.schedule_sharded(inst, G)
        r = dts.schedule_sharded(inst, G)[0]
        nx = max(r.prof_cycles[13], 1)
        print(f"{inst.name} G={G}: loop {r.loop_ms:.2f} ms, {r.n_served} dec, {r.n_scans} scans, "
              f"{r.prof_cycles[13]} exchanges, {r.prof_cycles[12] / nx:.0f} cyc/exchange, "
              f"{1e6 * r.loop_ms / max(r.n_scans, 1):.0f} ns/scan", flush=True)
