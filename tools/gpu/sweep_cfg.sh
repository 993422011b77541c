# C5 sweep launch configuration: CTA size x shared-memory share per CTA.
O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for B in 256 128 64; do for D in 4 6 8; do
  DTS_BLOCK=$B DTS_SWEEP_SMEM_DIV=$D timeout 300 python bench.py --workload C5 --steps 3 --warmup 3 --no-cpu-baseline > $O/sw_${B}_${D}.json 2>$O/sw_${B}_${D}.err
  python -c "import json;d=json.load(open('$O/sw_${B}_${D}.json'));print('block $B div $D', round(d['ms_per_step'],1), 'ms', round(d['value']/1e6,1), 'M dec/s')"
done; done
