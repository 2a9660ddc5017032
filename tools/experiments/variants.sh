mkdir -p gpurun_out
for lib in tile8 tile16; do for u in 16384 65536; do echo -n "$lib "; AP_LIB_PATH=build/variants/lib_$lib.so timeout 120 python tools/prof_hit.py $u 8; done; done > gpurun_out/variants.txt 2>&1
