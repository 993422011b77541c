TAG=${1:-src}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "fetch or sweep or config2 or compact" > $O/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest.log
for i in 1 2; do timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/${TAG}_c2_$i.json 2>$O/${TAG}_c2_$i.err
python -c "import json;d=json.load(open('$O/${TAG}_c2_$i.json'));print('C2', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M dec/s; e2e', round(d['e2e']['value']/1e6,2))"; done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dts_cta_kernel -s 1 -c 1 -o $O/${TAG}_c2n100 python tools/one_instance.py C2 19 > $O/${TAG}_ncu.log 2>&1; echo "ncu rc=$?"
ncu -i $O/${TAG}_c2n100.ncu-rep --page source --csv --print-source sass > $O/${TAG}_sass.csv 2>&1
ncu -i $O/${TAG}_c2n100.ncu-rep --page source --csv > $O/${TAG}_srccuda.csv 2>&1
ls -la $O/${TAG}_*
