# per-access dereference with a out-of-line miss path (measurement build) vs the product (__activemask per access)
mkdir -p gpurun_out/mnl; O=gpurun_out/mnl
for i in 1 2; do
for v in prod mn; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  AP_DEREF_GRIDS=148 AP_FIG6_TBS=148 timeout 600 python tools/exp_hit.py 2>&1 | grep -E "deref|16B (read|add)" | sed "s/^/$v /" >> $O/res.txt
done
done
cat $O/res.txt
