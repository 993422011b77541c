# C2 (headline) batch: CTA size per instance.
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for B in 32 64 96 128 256; do
  DTS_BLOCK=$B timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/c2b_${B}.json 2>$O/c2b_${B}.err
  python -c "import json;d=json.load(open('$O/c2b_${B}.json'));print('C2 block $B', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,2), 'M dec/s')"
done
for B in 32 64 128 256 512; do
  DTS_BLOCK=$B timeout 300 python bench.py --workload C3 --steps 5 --warmup 3 --no-cpu-baseline > $O/c3b_${B}.json 2>$O/c3b_${B}.err
  python -c "import json;d=json.load(open('$O/c3b_${B}.json'));print('C3 block $B', round(d['ms_per_step'],3), 'ms', round(d['value']/1e6,3), 'M dec/s')"
done
