# bench.py lines (C1, C2, C4) for the default library and each build/variants/lib_*.so
mkdir -p gpurun_out
for v in default $(ls build/variants 2>/dev/null | sed -n 's/^lib_\(.*\)\.so$/\1/p'); do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  for w in ${WORKLOADS:-c1 c2 c4}; do
    AP_LIB_PATH=$L timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bv_${v}_$w.json 2> gpurun_out/bv_${v}_$w.err
    python - "$v" "$w" <<'PY'
import json, sys
v, w = sys.argv[1:]
d = json.load(open(f"gpurun_out/bv_{v}_{w}.json"))
fb = d.get("fault_bound", {})
print(v, w, d["value"], d["unit"], "frac", d["roofline"]["frac"], "hit_ratio", fb.get("hit_ratio"),
      "evict", fb.get("evictions"), "waits", fb.get("waits"), "nofree", fb.get("nofree"))
PY
  done
done
