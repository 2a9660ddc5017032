# C1 (64 frames, 148 warps, work queue, drop-behind): fault-path back-off and sweep-length sweep
mkdir -p gpurun_out/c1b; O=gpurun_out/c1b/res.txt
P=$(python -c "import paper_conf_isca_shaharbs16_b200 as ap; print(ap.AP_SEQ_QUEUE)")
for b in 64,4096 256,4096 1024,4096 64,16384 256,16384 1024,16384 1024,65536 4096,65536 16384,65536; do
  echo "== backoff $b" >> $O
  AP_EXP_PATTERN=$P AP_EXP_FRAMES=64 AP_EXP_GRIDS=148 AP_EXP_BACKOFF=$b timeout 120 python tools/exp_c1.py >> $O 2>&1
done
for s in 1 2 3 5; do
  echo "== sweep $s (backoff default)" >> $O
  AP_EXP_PATTERN=$P AP_EXP_FRAMES=64 AP_EXP_GRIDS=148 AP_EXP_SWEEP=$s timeout 120 python tools/exp_c1.py >> $O 2>&1
  echo "== sweep $s backoff 1024,16384" >> $O
  AP_EXP_PATTERN=$P AP_EXP_FRAMES=64 AP_EXP_GRIDS=148 AP_EXP_SWEEP=$s AP_EXP_BACKOFF=1024,16384 timeout 120 python tools/exp_c1.py >> $O 2>&1
done
echo "== grid 64 reference" >> $O
AP_EXP_PATTERN=$P AP_EXP_FRAMES=64 AP_EXP_GRIDS=64 timeout 120 python tools/exp_c1.py >> $O 2>&1
cat $O
