# tests + state/edge A/B + C2 block sizes + C5 split sweep.  usage: bash tools/gpu/next.sh TAG
TAG=${1:-nx}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -4 $O/${TAG}_pytest_gpu.log
timeout 600 python tools/ab_state.py c2 c3 c5long 2>&1 | tee $O/${TAG}_ab.txt
for B in 32 64 128; do
  DTS_BLOCK=$B timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/${TAG}_c2b_${B}.json 2>$O/${TAG}_c2b_${B}.err
  python -c "import json;d=json.load(open('$O/${TAG}_c2b_${B}.json'));print('C2 block $B', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M dec/s')"
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/${TAG}_c2.json 2>$O/${TAG}_c2.err
python -c "import json;d=json.load(open('$O/${TAG}_c2.json'));print('C2 auto', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M dec/s')"
for SB in 64 128 0; do
  DTS_SWEEP_SMALL_BLOCK=$SB timeout 300 python bench.py --workload C5 --steps 3 --warmup 3 --no-cpu-baseline > $O/${TAG}_c5_$SB.json 2>$O/${TAG}_c5_$SB.err
  python -c "import json;d=json.load(open('$O/${TAG}_c5_$SB.json'));print('C5 small_block $SB', round(d['ms_per_step'],1), 'ms', round(d['value']/1e6,1), 'M dec/s')"
done
timeout 300 python tools/san_c5.py 12 > $O/${TAG}_rep.log 2>&1; echo "C5 rep x12 rc=$?"; tail -1 $O/${TAG}_rep.log
DTS_BLOCK=128 timeout 300 python tools/san_c5.py 20 > $O/${TAG}_rep128.log 2>&1; echo "C5 rep block128 x20 rc=$?"; tail -1 $O/${TAG}_rep128.log
DTS_BLOCK=128 timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_c5.py 1 16 > $O/${TAG}_sync.log 2>&1; echo "synccheck rc=$?"; grep -v "^=========     " $O/${TAG}_sync.log | tail -5
