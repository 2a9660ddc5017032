# N4 ablation with the hash build passing parity: hash-table page table vs the dense PTE array (same bench, AP_LIB_PATH selects the library)
mkdir -p gpurun_out/hab; O=gpurun_out/hab
timeout 900 python -m pytest tests/test_gpu_pt_hash.py -q -p no:cacheprovider 2>&1 | tail -1 > $O/test.txt; cat $O/test.txt
for lib in libapointer.so libapointer_hash.so; do
  export AP_LIB_PATH=$PWD/paper_conf_isca_shaharbs16_b200/$lib
  timeout 900 python bench.py --no-collage --no-reads --no-c5 --no-cpu-baseline > $O/c2_$lib.json 2>$O/c2_$lib.err
  timeout 600 python bench.py --workload c4 --no-cpu-baseline > $O/c4_$lib.json 2>$O/c4_$lib.err
  timeout 600 python bench.py --workload c3 --no-cpu-baseline > $O/c3_$lib.json 2>$O/c3_$lib.err
  python - >> $O/res.txt <<PY
import json
d = json.load(open("$O/c2_$lib.json")); h = d["hit"]; m = d["minor"]
c4 = json.load(open("$O/c4_$lib.json")); c3 = json.load(open("$O/c3_$lib.json"))
print("$lib", "C2 fills GB/s", d["roofline"]["achieved"], "frac", d["roofline"]["frac"],
      "| hit tile GB/s", h["apointer_GBps"], "vs raw", h["overhead_vs_raw"],
      "| per-access", h["access_styles"]["deref"]["GBps"], "vs raw twin", h["deref_vs_raw_per_access_twin"]["overhead"],
      "| M2r G reads/s", round(m["reads_per_s"] / 1e9, 2), "| C3 fills", c3["value"], "| C4 ms", c4["ms_per_step"],
      "| resident g8", c4["collage"].get("resident_cache", {}).get("group8"))
PY
done
unset AP_LIB_PATH
cat $O/res.txt
