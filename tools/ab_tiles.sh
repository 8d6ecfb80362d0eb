# A/B of the tile-shared scan against the item path on the bench workloads (development aid)
for w in ${WORKLOADS:-C2a C2b}; do
  for v in ${VARIANTS:-default items}; do
    if [ "$v" = default ]; then env=""; elif [ "$v" = items ]; then env="OLAP_NO_TILES=1"; else env="OLAP_LIB=variants/$v.so"; fi
    env $env python bench.py --no-cpu-baseline --workload $w --e2e-steps 1 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w $v', round(d['value']), round(d['roofline']['achieved']))"
  done
done
