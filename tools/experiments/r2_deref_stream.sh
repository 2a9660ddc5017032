# per-access dereference: one ring across the warp's units (prod) vs a ring per unit (ds0)
mkdir -p gpurun_out/dstr; O=gpurun_out/dstr
timeout 900 python -m pytest tests/test_gpu_reads.py tests/test_gpu_compute.py -q -x > $O/t.txt 2>&1; tail -1 $O/t.txt >> $O/res.txt
for i in 1 2; do
for v in prod ds0; do
  if [ $v = prod ]; then unset AP_LIB_PATH; else export AP_LIB_PATH=$PWD/build/variants/lib_$v.so; fi
  AP_DEREF_GRIDS=148,296 AP_FIG6_TBS=148 timeout 600 python tools/exp_hit.py 2>&1 | sed "s/^/$v /" >> $O/res.txt
done
done
cat $O/res.txt
