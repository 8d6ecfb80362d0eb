# A/B of differently-compiled builds (variants/<v>.so) on bench workloads: VARIANTS, WORKLOADS, EXTRA
mkdir -p gpurun_out
for w in ${WORKLOADS:-C5}; do
  for v in ${VARIANTS:-default}; do
    if [ "$v" = default ]; then env=""; else env="OLAP_LIB=variants/$v.so"; fi
    env $env timeout 600 python bench.py --no-cpu-baseline --workload $w --e2e-steps 0 ${EXTRA:-} 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w $v ${EXTRA:-}', round(d['value']), round(d['roofline']['achieved']))" >> gpurun_out/ab.txt 2>&1
  done
done
