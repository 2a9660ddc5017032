# hash-table build vs the read + collage parity suites (current code), 2 s watchdog so a deadlock cannot stall the run
mkdir -p gpurun_out/hs2; O=gpurun_out/hs2
AP_TIMEOUT_MS=2000 AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 1200 python -m pytest tests/test_gpu_reads.py tests/test_gpu_collage.py -q -p no:cacheprovider -rf > $O/suite.txt 2>&1; echo "rc=$?" >> $O/suite.txt
tail -25 $O/suite.txt
