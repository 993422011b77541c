import sys; sys.path.insert(0,'.'); sys.path.insert(0,'tests')
import gen, oracle, paper_conf_ipps_gonthiermt22_b200 as dts
from parity import assert_parity
for inst in [gen.fig1(), gen.random_shared(300, 64, 3, M=8, K=3, seed=7), gen.matmul2d(12, M=5, K=2)]:
    bus = 10**9 if inst.name=='fig1' else oracle.DEFAULT_BUS_BPS
    g = dts.schedule(inst, bus_bps=bus, block_threads=64)
    o = oracle.run(inst, bus_bps=bus)
    try:
        assert_parity(g, o); print(inst.name, 'OK')
    except AssertionError as e:
        print(inst.name, 'FAIL', e); print(g.orders()); print(o.orders())
