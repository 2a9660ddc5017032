# NEXT N4 prefetch ablation (Table I): the default library
# (speculative load issued with the vote), lib_nospec (load after the vote),
# lib_pf2 (speculative + stride prefetch 2 steps ahead into L2).
# Needs build/variants/lib_{nospec,pf2}.so.
for v in default nospec pf2; do
  if [ $v = default ]; then L=paper_conf_isca_shaharbs16_b200/libapointer.so; else L=build/variants/lib_$v.so; fi
  echo "=== $v"
  AP_LIB_PATH=$L timeout 120 python tools/latency.py | grep -A3 "page=4096"
  for g in 148 592; do echo "-- per-access 16-B hit read, grid $g x 512"; AP_GRID=$g AP_LIB_PATH=$L timeout 300 python tools/prof_hit.py 65536 4 | grep deref; done
  echo "-- uniform-random 4-B reads, resident 1 GiB (every read a minor fault)"
  AP_LIB_PATH=$L timeout 300 python tools/prof_minor.py
done
