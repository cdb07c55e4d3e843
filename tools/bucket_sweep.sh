# Query-bucketing sweep (1 GPU): configs x (off / plain bucketed / bucket-local directory) x slice.
mkdir -p gpurun_out
out=gpurun_out/bucket_sweep.log
: > $out
for c in ${CONFIGS:-c3 c5 c2}; do
  for b in ${VARIANTS:-"0 16777216 0" "1 16777216 0" "1 16777216 1" "1 4194304 1" "1 1048576 1"}; do
    set -- $b
    echo "== $c bucket=$1 slice=$2 items=$3" >> $out
    timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 \
      --bucket $1 --bucket-slice $2 --bucket-items $3 > gpurun_out/bs.log 2>&1
    tail -1 gpurun_out/bs.log | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])" >> $out 2>&1 || tail -3 gpurun_out/bs.log >> $out
  done
done
cat $out
