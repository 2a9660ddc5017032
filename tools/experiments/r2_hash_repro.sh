# hash build: the unaligned 40-frame collage cases alone (60 s each)
mkdir -p gpurun_out/hr; O=gpurun_out/hr
for k in "40-4-1" "40-2-1 or 40-4-1" "40-8-1"; do
  AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 60 python -m pytest tests/test_gpu_collage.py -k "unaligned and ($k)" -q -x -p no:cacheprovider > $O/t.txt 2>&1; echo "[$k] rc=$? $(tail -1 $O/t.txt)" >> $O/res.txt
done
AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 120 python -m pytest tests/test_gpu_collage.py -k "unaligned or slices" -q -x -p no:cacheprovider > $O/t2.txt 2>&1; echo "[slices+unaligned] rc=$? $(tail -1 $O/t2.txt)" >> $O/res.txt
cat $O/res.txt
