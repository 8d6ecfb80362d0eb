set -u
mkdir -p gpurun_out
OUT=gpurun_out/vw_${TAG:-r02vw4}.txt
for w in C2a C3 C5; do
  for v in 1 2 4 8; do
    if [ $v = 1 ]; then unset OLAP_BENCH_VIRTUAL_WORLD; else export OLAP_BENCH_VIRTUAL_WORLD=$v; fi
    timeout 900 python bench.py --workload $w --no-cpu-baseline --e2e-steps 0 > gpurun_out/${TAG:-r02vw4}_${w}_$v.log 2>&1
    tail -1 gpurun_out/${TAG:-r02vw4}_${w}_$v.log > gpurun_out/${TAG:-r02vw4}_${w}_$v.jsonl
    python -c "import json; d=json.loads(open('gpurun_out/${TAG:-r02vw4}_${w}_$v.jsonl').read()); print('$w V=$v', round(d['value']), round(d['ms_per_step'],3), d['scaling'])" >> $OUT 2>&1
  done
done
echo done
