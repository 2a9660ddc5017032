mkdir -p gpurun_out/db; O=gpurun_out/db
t0=$(date +%s); timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err; echo "rc=$? default bench wall $(( $(date +%s) - t0 )) s" > $O/res.txt
t0=$(date +%s); timeout 600 python bench.py --impl reference > $O/ref.json 2> $O/ref.err; echo "rc=$? reference wall $(( $(date +%s) - t0 )) s" >> $O/res.txt
cat $O/res.txt; tail -3 $O/bench.err
