# Round measurement: tests, bench lines for every config, reference arm, ncu launch list + full captures.
# usage (on the GPU box): bash tools/gpu/measure.sh TAG
TAG=${1:-r01f}
O=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $O/${TAG}_bench_C2.json 2> $O/${TAG}_bench_C2.err; echo "C2 rc=$?"
for W in C1 C3; do timeout 600 python bench.py --workload $W > $O/${TAG}_bench_$W.json 2> $O/${TAG}_bench_$W.err; echo "$W rc=$?"; done
timeout 900 python bench.py --workload C5 --steps 5 > $O/${TAG}_bench_C5.json 2> $O/${TAG}_bench_C5.err; echo "C5 rc=$?"
for W in C4a C4b; do timeout 900 python bench.py --workload $W --steps 3 --warmup 3 > $O/${TAG}_bench_$W.json 2> $O/${TAG}_bench_$W.err; echo "$W rc=$?"; done
timeout 600 python bench.py --workload C3 --shards 4 --steps 5 --no-cpu-baseline > $O/${TAG}_bench_C3_shards4.json 2>&1; echo "C3s rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/${TAG}_bench_reference_C2.json 2> $O/${TAG}_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_C2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_bench.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:dts_cta_kernel -s 3 -c 1 -o $O/${TAG}_full_C2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C2.log 2>&1; echo "full C2 rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:dts_cta_kernel -s 6 -c 2 -o $O/${TAG}_full_C5 python bench.py --workload C5 --steps 1 --warmup 3 --no-cpu-baseline > $O/${TAG}_ncu_full_C5.log 2>&1; echo "full C5 rc=$?"
ls $O | grep $TAG
DTS_BLOCK=256 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/${TAG}_c2_b256.json 2>/dev/null; python -c "import json;d=json.load(open(\"$O/${TAG}_c2_b256.json\"));print(\"C2 block 256\", d[\"ms_per_step\"], d[\"value\"])"
