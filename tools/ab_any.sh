# A/B of variants/<v>.so vs the default build on any workload, printing q/s only (VARIANTS, WORKLOADS, EXTRA)
mkdir -p gpurun_out
for w in ${WORKLOADS:-T}; do
  for v in ${VARIANTS:-head default}; do
    if [ "$v" = default ]; then env=""; else env="OLAP_LIB=variants/$v.so"; fi
    env $env timeout 600 python bench.py --no-cpu-baseline --workload $w --e2e-steps 1 ${EXTRA:-} 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w $v ${EXTRA:-}', round(d['value']))" >> gpurun_out/ab.txt 2>&1
  done
done
