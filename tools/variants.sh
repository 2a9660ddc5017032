mkdir -p gpurun_out
for v in "512 1 8 148" "256 3 8 444" "512 2 4 296"; do set -- $v; tag=t$1_b$2_tile$3
 for u in 16384 65536; do echo -n "$tag "; AP_LIB_PATH=build/variants/lib_$tag.so AP_GRID=$4 AP_BLOCK=$1 timeout 120 python tools/prof_hit.py $u 8; done
done > gpurun_out/variants.txt 2>&1
