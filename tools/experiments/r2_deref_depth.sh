# per-access dereference ring depth D = 8 (product) / 12 / 16: apointer vs raw per-access twin
mkdir -p gpurun_out/dd; O=gpurun_out/dd; : > $O/res.txt
for i in 1 2; do
for v in prod d12 d16; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  AP_DEREF_GRIDS=148 AP_FIG6_TBS=148 timeout 600 python tools/exp_hit.py 2>&1 | grep -E "deref grid" | sed "s/^/$v /" >> $O/res.txt
done
done
cat $O/res.txt
