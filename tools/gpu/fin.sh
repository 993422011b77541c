TAG=${1:-fin}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
for i in 1 2; do timeout 300 python bench.py > $O/${TAG}_bench_C2_$i.json 2> $O/${TAG}_bench_C2_$i.err; python -c "import json;d=json.load(open('$O/${TAG}_bench_C2_$i.json'));print('C2', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M/s e2e', round(d['e2e']['value']/1e6,2), d['clocks'])"; done
timeout 300 python bench.py --workload C1 > $O/${TAG}_bench_C1.json 2> $O/${TAG}_bench_C1.err; python -c "import json;d=json.load(open('$O/${TAG}_bench_C1.json'));print('C1', d['value'], d['e2e']['value'], d['clocks'])"
