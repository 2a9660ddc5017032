# hash-table page table build against the read + collage parity suites (per-test limit 60 s)
mkdir -p gpurun_out/hs; O=gpurun_out/hs
AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/libapointer_hash.so timeout 900 python -m pytest tests/test_gpu_reads.py tests/test_gpu_collage.py -q -x -p no:cacheprovider --timeout 60 -v > $O/suite.txt 2>&1; echo "rc=$?" >> $O/suite.txt
grep -E "PASSED|FAILED|ERROR|Timeout|rc=" $O/suite.txt | tail -8
grep -c PASSED $O/suite.txt
