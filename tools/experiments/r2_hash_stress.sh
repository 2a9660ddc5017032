# hash-table build against the random collage cases, one process per case (60 s each), 2 s watchdog
mkdir -p gpurun_out/hst; O=gpurun_out/hst; : > $O/res.txt
for c in $(seq 0 15); do
  AP_STRESS_CASES=$c-$((c+1)) AP_TIMEOUT_MS=2000 AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 60 python -m pytest tests/test_gpu_collage_stress.py -q -p no:cacheprovider > $O/t.txt 2>&1
  echo "case $c rc=$? $(tail -1 $O/t.txt | cut -c1-80)" >> $O/res.txt
done
python -c "
import sys; sys.path.insert(0,'tests'); import test_gpu_collage_stress as t
for c in range(16): print(c, t._cfg(c))" >> $O/res.txt 2>&1
cat $O/res.txt
