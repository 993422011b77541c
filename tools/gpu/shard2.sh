python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_shard.py -x -q > gpurun_out/shard.log 2>&1; echo "shard rc=$?"
tail -5 gpurun_out/shard.log
for S in 1 2 4 8; do
  timeout 300 python bench.py --workload C3 --shards $S --steps 3 --warmup 1 --no-cpu-baseline > gpurun_out/b_C3_s$S.json 2>gpurun_out/b_C3_s$S.err
  python -c "import json;d=json.load(open('gpurun_out/b_C3_s$S.json'));print('C3 shards $S', d['value'], d['ms_per_step'])"
done
for S in 1 4 16; do
  timeout 300 python bench.py --workload C4b --shards $S --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/b_C4b_s$S.json 2>gpurun_out/b_C4b_s$S.err
  python -c "import json;d=json.load(open('gpurun_out/b_C4b_s$S.json'));print('C4b shards $S', d['value'], d['ms_per_step'])"
done
