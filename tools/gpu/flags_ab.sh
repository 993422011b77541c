# same-box A/B of nvcc cache-operator flags, then the final round check
O=gpurun_out
for r in 1 2; do
for L in tools/var/v_base.so tools/var/v_cg.so tools/var/v_wt.so; do
  timeout 300 python tools/lib_ab.py $L 9 2>&1 | tail -1
done; done | tee $O/r01n_lib_ab_flags.txt
bash tools/gpu/final.sh r01n
