TAG=${1:-fin2}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 300 python tools/e2e_phases.py C2
timeout 600 python tools/e2e_phases.py C5
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
timeout 300 python bench.py > $O/${TAG}_bench_C2.json 2> $O/${TAG}_bench_C2.err; python -c "import json;d=json.load(open('$O/${TAG}_bench_C2.json'));print('C2', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M/s e2e', round(d['e2e']['value']/1e6,2), d['clocks'])"
timeout 900 python bench.py --workload C5 --steps 5 > $O/${TAG}_bench_C5.json 2> $O/${TAG}_bench_C5.err; python -c "import json;d=json.load(open('$O/${TAG}_bench_C5.json'));print('C5', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M/s e2e', round(d['e2e']['value']/1e6,2), d['clocks'])"
