# per-GPU step of V-GPU weak-scaling jobs (default shard blocks), shard 0 and other shards for balance
set -u
mkdir -p gpurun_out
OUT=gpurun_out/vw_r02vw3.txt
for w in C5 C2a; do
  for v in 1 2 4 8; do
    if [ $v = 1 ]; then unset OLAP_BENCH_VIRTUAL_WORLD; else export OLAP_BENCH_VIRTUAL_WORLD=$v; fi
    export OLAP_BENCH_VIRTUAL_SHARD=0
    timeout 600 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 > gpurun_out/vw3_${w}_$v.log 2>&1
    tail -1 gpurun_out/vw3_${w}_$v.log > gpurun_out/vw3_${w}_$v.jsonl
    python -c "import json; d=json.loads(open('gpurun_out/vw3_${w}_$v.jsonl').read()); print('$w V=$v g=0', round(d['value']), round(d['ms_per_step'],3))" >> $OUT 2>&1
  done
  export OLAP_BENCH_VIRTUAL_WORLD=8
  for g in 3 7; do
    export OLAP_BENCH_VIRTUAL_SHARD=$g
    timeout 600 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w V=8 g=$g', round(d['value']), round(d['ms_per_step'],3))" >> $OUT 2>&1
  done
done
echo done
