# hit-mode SEQ kernels (tile / range / deref access styles): library variants
# lib_seqN.so (k_seq built for N CTAs of 512 threads per SM) at grid 148*N
mkdir -p gpurun_out
for v in default $(ls build/variants 2>/dev/null | sed -n 's/^lib_\(.*\)\.so$/\1/p'); do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; n=1; else L=build/variants/lib_$v.so; n=${v#seq}; fi
  echo "== $v grid $((148*n))"; AP_GRID=$((148*n)) AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 4
done > gpurun_out/seq_variants.txt 2>&1
cat gpurun_out/seq_variants.txt
