# hash-table build without the post-probe __syncwarp(m), against the read, collage and random collage parity suites (2 s watchdog, bounded)
mkdir -p gpurun_out/hfx; O=gpurun_out/hfx
AP_TIMEOUT_MS=2000 AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 1200 python -m pytest tests/test_gpu_reads.py tests/test_gpu_collage.py tests/test_gpu_collage_stress.py -q -p no:cacheprovider -rf > $O/suite.txt 2>&1; r=$?; echo "rc=$r" >> $O/suite.txt
tail -15 $O/suite.txt
AP_STRESS_CASES=12-112 AP_TIMEOUT_MS=2000 AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 900 python -m pytest tests/test_gpu_collage_stress.py -q -p no:cacheprovider > $O/soak.txt 2>&1; r=$?; echo "rc=$r" >> $O/soak.txt
tail -3 $O/soak.txt
